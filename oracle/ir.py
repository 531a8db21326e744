"""Oracle-side parser for the IR v1 text format.

Test infrastructure only (see oracle/__init__.py).  Written independently of
the C++ parser in paper_conf_ipps_jiw21_b200/csrc; the two share only the
format specification.

The IR stands in for the paper's GPU assembly (Figs 2-6 list GCN-style
instructions ``XOR r3, r4, 0xF`` ...): registers, one result per
instruction (R-12), uniform control flow, explicit memory operands.
"""
from __future__ import annotations

import re
from dataclasses import dataclass, field

VECTOR_SPECIALS = ("tid", "laneid")
UNIFORM_SPECIALS = ("ntid", "ctaid", "nctaid", "warpid", "nwarps")

ALU2 = {"iadd", "isub", "imul", "and", "or", "xor", "shl", "shr", "sar",
        "rotl", "rotr", "umin", "umax", "imin", "imax", "fadd", "fsub", "fmul"}
ALU1 = {"mov", "not", "neg", "i2f", "u2f", "f2i"}
ALU3 = {"ffma", "imad", "sel"}
SETP_CMPS = ("eq", "ne", "lt", "le", "gt", "ge")
SETP_TYPES = ("u", "s", "f")


class IRError(ValueError):
    pass


@dataclass(frozen=True)
class Opd:
    """An operand.  kind: 'v' / 's' register, 'imm' (u32), 'sp' special."""
    kind: str
    val: object  # int for v/s/imm, str for sp

    @property
    def is_reg(self):
        return self.kind in ("v", "s")

    @property
    def reg(self):
        return f"{self.kind}{self.val}" if self.is_reg else None


@dataclass
class Instr:
    op: str                      # opcode (setp carries cmp/type in `mod`)
    dst: Opd | None = None       # result register or None (stg, atom _, control)
    srcs: list = field(default_factory=list)   # value operands (registers/imm/specials)
    buf: str | None = None       # memory buffer name (ldg/stg/atom)
    idx: Opd | None = None       # memory index operand (element index, u32 words)
    guard: Opd | None = None     # '@reg' lane guard for memory ops
    target: str | None = None    # branch label
    mod: tuple = ()              # setp: (cmp, type)
    line: int = 0
    text: str = ""

    def uses(self):
        """Registers read, in operand order (duplicates kept)."""
        out = []
        for o in self.srcs:
            if o.is_reg:
                out.append(o.reg)
        if self.idx is not None and self.idx.is_reg:
            out.append(self.idx.reg)
        if self.guard is not None and self.guard.is_reg:
            out.append(self.guard.reg)
        return out

    @property
    def defreg(self):
        return self.dst.reg if self.dst is not None else None


@dataclass
class Program:
    name: str
    buffers: dict            # name -> 'ro' | 'rw' | 'wo'  (insertion ordered)
    uniforms: list           # names of u32 kernel parameters
    nv: int
    ns: int
    block: int
    instrs: list             # Instr, global program order (poll markers removed)
    bbs: list                # list of (start, end) half-open global index ranges
    labels: dict             # label -> bb index
    explicit_sites: list     # global instruction indices with a 'poll' before them
    bb_succ: list = field(default_factory=list)
    smem: int = 0            # u32 words of shared memory per block (N2)

    @property
    def has_barriers(self):
        return any(i.op == "bar" for i in self.instrs)

    @property
    def nwarps(self):
        return self.block // 32

    def bb_of(self, i):
        for b, (s, e) in enumerate(self.bbs):
            if s <= i < e:
                return b
        raise IndexError(i)

    def is_vector(self, reg):
        return reg[0] == "v"

    def all_regs(self):
        return [f"v{i}" for i in range(self.nv)] + [f"s{i}" for i in range(self.ns)]


_num = re.compile(r"^-?(0x[0-9a-fA-F]+|\d+)$")
_fbits = re.compile(r"^0f[0-9a-fA-F]{8}$")
_mem = re.compile(r"^([A-Za-z_]\w*)\[(.+)\]$")


def _parse_opd(tok, uniforms, line):
    tok = tok.strip()
    if re.fullmatch(r"v\d+", tok):
        return Opd("v", int(tok[1:]))
    if re.fullmatch(r"s\d+", tok):
        return Opd("s", int(tok[1:]))
    if _fbits.match(tok):
        return Opd("imm", int(tok[2:], 16))
    if _num.match(tok):
        neg = tok.startswith("-")
        t = tok[1:] if neg else tok
        v = int(t, 16) if t.lower().startswith("0x") else int(t)
        if neg:
            v = -v
        if not (-(1 << 31) <= v < (1 << 32)):
            raise IRError(f"line {line}: immediate out of range: {tok}")
        return Opd("imm", v & 0xFFFFFFFF)
    if tok.startswith("%"):
        name = tok[1:]
        if name in VECTOR_SPECIALS or name in UNIFORM_SPECIALS or name in uniforms:
            return Opd("sp", name)
        raise IRError(f"line {line}: unknown special {tok}")
    raise IRError(f"line {line}: bad operand {tok!r}")


def is_uniform_opd(o):
    return o.kind in ("s", "imm") or (o.kind == "sp" and o.val not in VECTOR_SPECIALS)


def parse(text: str) -> Program:
    name = None
    buffers: dict = {}
    uniforms: list = []
    nv = ns = None
    block = None
    smem = 0
    body = []  # (lineno, str)
    for ln, raw in enumerate(text.splitlines(), 1):
        s = raw.split("#", 1)[0].strip()
        if not s:
            continue
        if s.startswith("."):
            parts = s.split()
            d = parts[0]
            if d == ".kernel" and len(parts) == 2:
                name = parts[1]
            elif d == ".buffer" and len(parts) == 3 and parts[1] in ("ro", "rw", "wo"):
                if parts[2] in buffers:
                    raise IRError(f"line {ln}: duplicate buffer {parts[2]}")
                if not re.fullmatch(r"[A-Za-z_]\w*", parts[2]):
                    raise IRError(f"line {ln}: bad buffer name")
                buffers[parts[2]] = parts[1]
            elif d == ".uniform" and len(parts) == 2:
                if parts[1] in VECTOR_SPECIALS or parts[1] in UNIFORM_SPECIALS or parts[1] in uniforms or \
                        not re.fullmatch(r"[A-Za-z_]\w*", parts[1]):
                    raise IRError(f"line {ln}: bad uniform name {parts[1]}")
                uniforms.append(parts[1])
            elif d == ".smem" and len(parts) == 2 and parts[1].isdigit():
                smem = int(parts[1])
                if smem > 12288:
                    raise IRError(f"line {ln}: .smem too large (max 12288 words)")
            elif d in (".vregs", ".sregs", ".block") and len(parts) == 2 and parts[1].isdigit():
                if len(parts[1]) > 6:
                    raise IRError(f"line {ln}: value too large")
                v = int(parts[1])
                if d == ".vregs":
                    nv = v
                elif d == ".sregs":
                    ns = v
                else:
                    block = v
            else:
                raise IRError(f"line {ln}: bad directive {s!r}")
            continue
        body.append((ln, s))
    if name is None or nv is None or ns is None or block is None:
        raise IRError("missing .kernel/.vregs/.sregs/.block")
    if block <= 0 or block % 32 or block > 1024:
        raise IRError(".block must be a positive multiple of 32, <= 1024")
    if nv > 4096 or ns > 4096:
        raise IRError("too many registers")

    instrs = []
    label_at = {}      # label -> global instr index where it starts
    poll_pending = False
    explicit_sites = []
    for ln, s in body:
        m = re.fullmatch(r"([A-Za-z_]\w*):", s)
        if m:
            lab = m.group(1)
            if lab in label_at:
                raise IRError(f"line {ln}: duplicate label {lab}")
            label_at[lab] = len(instrs)
            continue
        if s == "poll":
            poll_pending = True
            continue
        ins = _parse_instr(s, ln, buffers, uniforms)
        if poll_pending:
            explicit_sites.append(len(instrs))
            poll_pending = False
        instrs.append(ins)
    if poll_pending:
        raise IRError("'poll' after the last instruction")
    if not instrs:
        raise IRError("empty kernel")

    # Basic blocks: leaders = 0, label targets, instruction after a terminator.
    leaders = {0}
    for lab, i in label_at.items():
        if i >= len(instrs):
            raise IRError(f"label {lab} at end of kernel")
        leaders.add(i)
    for i, ins in enumerate(instrs):
        if ins.op in ("bra", "brnz", "brz", "exit") and i + 1 < len(instrs):
            leaders.add(i + 1)
    ls = sorted(leaders)
    bbs = [(ls[k], ls[k + 1] if k + 1 < len(ls) else len(instrs)) for k in range(len(ls))]
    start_to_bb = {s0: b for b, (s0, _) in enumerate(bbs)}
    labels = {lab: start_to_bb[i] for lab, i in label_at.items()}
    if instrs[-1].op not in ("bra", "exit"):
        raise IRError("the last instruction must be 'bra' or 'exit'")

    prog = Program(name, buffers, uniforms, nv, ns, block, instrs, bbs, labels, explicit_sites)
    prog.smem = smem
    # validate registers / typing, successors
    succ = []
    for b, (s0, e0) in enumerate(bbs):
        last = instrs[e0 - 1]
        out = []
        if last.op in ("bra", "brnz", "brz"):
            if last.target not in labels:
                raise IRError(f"line {last.line}: unknown label {last.target}")
            if last.op != "bra":
                out.append(b + 1)
            out.append(labels[last.target])
        elif last.op != "exit":
            out.append(b + 1)
        succ.append(sorted(set(out)))
    prog.bb_succ = succ
    for ins in instrs:
        _validate(prog, ins)
    if any(i.op in ("lds", "sts") for i in instrs) and not prog.has_barriers:
        raise IRError("kernels using shared memory must synchronise with 'bar' "
                      "(their preemption is block-uniform at barriers)")
    if prog.has_barriers:
        for c in explicit_sites:
            if instrs[c].op != "bar":
                raise IRError(f"line {instrs[c].line}: in a kernel with barriers, 'poll' may only precede 'bar' "
                              "(preemption is block-uniform at barriers)")
    return prog


def _split_ops(rest):
    out, depth, cur = [], 0, ""
    for ch in rest:
        if ch == "[":
            depth += 1
        elif ch == "]":
            depth -= 1
        if ch == "," and depth == 0:
            out.append(cur.strip())
            cur = ""
        else:
            cur += ch
    if cur.strip():
        out.append(cur.strip())
    return out


def _parse_instr(s, ln, buffers, uniforms):
    guard = None
    if s.startswith("@"):
        parts = s.split(None, 1)
        if len(parts) != 2:
            raise IRError(f"line {ln}: bad guard")
        g, s = parts
        guard = _parse_opd(g[1:], uniforms, ln)
        if not guard.is_reg:
            raise IRError(f"line {ln}: guard must be a register")
    parts = s.split(None, 1)
    opc = parts[0]
    ops = _split_ops(parts[1]) if len(parts) > 1 else []
    P = lambda t: _parse_opd(t, uniforms, ln)

    def mem(t):
        m = _mem.match(t.replace(" ", ""))
        if not m:
            raise IRError(f"line {ln}: expected BUF[idx], got {t!r}")
        if m.group(1) not in buffers:
            raise IRError(f"line {ln}: unknown buffer {m.group(1)}")
        return m.group(1), P(m.group(2))

    def dstreg(t):
        o = P(t)
        if not o.is_reg:
            raise IRError(f"line {ln}: destination must be a register")
        return o

    ins = None
    if opc.startswith("setp."):
        bits = opc.split(".")
        if len(bits) != 3 or bits[1] not in SETP_CMPS or bits[2] not in SETP_TYPES or len(ops) != 3:
            raise IRError(f"line {ln}: bad setp {s!r}")
        ins = Instr("setp", dstreg(ops[0]), [P(ops[1]), P(ops[2])], mod=(bits[1], bits[2]))
    elif opc in ALU2:
        if len(ops) != 3:
            raise IRError(f"line {ln}: {opc} takes 3 operands")
        ins = Instr(opc, dstreg(ops[0]), [P(ops[1]), P(ops[2])])
    elif opc in ALU1:
        if len(ops) != 2:
            raise IRError(f"line {ln}: {opc} takes 2 operands")
        ins = Instr(opc, dstreg(ops[0]), [P(ops[1])])
    elif opc in ALU3:
        if len(ops) != 4:
            raise IRError(f"line {ln}: {opc} takes 4 operands")
        ins = Instr(opc, dstreg(ops[0]), [P(ops[1]), P(ops[2]), P(ops[3])])
    elif opc == "ldg":
        if len(ops) != 2:
            raise IRError(f"line {ln}: ldg d, BUF[idx]")
        b, ix = mem(ops[1])
        ins = Instr("ldg", dstreg(ops[0]), [], buf=b, idx=ix)
    elif opc == "stg":
        if len(ops) != 2:
            raise IRError(f"line {ln}: stg BUF[idx], a")
        b, ix = mem(ops[0])
        ins = Instr("stg", None, [P(ops[1])], buf=b, idx=ix)
    elif opc in ("atom.add", "atom.cas"):
        n = 3 if opc == "atom.add" else 4
        if len(ops) != n:
            raise IRError(f"line {ln}: bad {opc}")
        d = None if ops[0] == "_" else dstreg(ops[0])
        b, ix = mem(ops[1])
        ins = Instr(opc, d, [P(t) for t in ops[2:]], buf=b, idx=ix)
    elif opc == "bra":
        if len(ops) != 1:
            raise IRError(f"line {ln}: bra LABEL")
        ins = Instr("bra", target=ops[0])
    elif opc in ("brnz", "brz"):
        if len(ops) != 2:
            raise IRError(f"line {ln}: {opc} s, LABEL")
        ins = Instr(opc, None, [P(ops[0])], target=ops[1])
    elif opc == "exit":
        if ops:
            raise IRError(f"line {ln}: exit takes no operands")
        ins = Instr("exit")
    elif opc == "bar":
        if ops:
            raise IRError(f"line {ln}: bar takes no operands")
        ins = Instr("bar")
    elif opc == "lds":
        if len(ops) != 2:
            raise IRError(f"line {ln}: lds d, idx")
        ins = Instr("lds", dstreg(ops[0]), [], buf="%smem", idx=P(ops[1]))
    elif opc == "sts":
        if len(ops) != 2:
            raise IRError(f"line {ln}: sts idx, a")
        ins = Instr("sts", None, [P(ops[1])], buf="%smem", idx=P(ops[0]))
    else:
        raise IRError(f"line {ln}: unknown opcode {opc!r}")
    if guard is not None and ins.op not in ("ldg", "stg", "atom.add", "atom.cas", "lds", "sts"):
        raise IRError(f"line {ln}: guards only on memory ops")
    ins.guard = guard
    ins.line = ln
    ins.text = s
    return ins


def _validate(prog, ins):
    ln = ins.line
    for o in list(ins.srcs) + [x for x in (ins.idx, ins.guard, ins.dst) if x is not None]:
        if o.kind == "v" and not (0 <= o.val < prog.nv):
            raise IRError(f"line {ln}: v{o.val} not declared")
        if o.kind == "s" and not (0 <= o.val < prog.ns):
            raise IRError(f"line {ln}: s{o.val} not declared")
    if ins.dst is not None and ins.dst.kind == "s":
        opds = list(ins.srcs) + ([ins.idx] if ins.idx is not None else []) + \
            ([ins.guard] if ins.guard is not None else [])
        if not all(is_uniform_opd(o) for o in opds):
            raise IRError(f"line {ln}: scalar destination needs uniform operands")
    if ins.op in ("brnz", "brz"):
        if ins.srcs[0].kind != "s":
            raise IRError(f"line {ln}: branch condition must be a scalar register")
    if ins.op in ("lds", "sts") and prog.smem == 0:
        raise IRError(f"line {ln}: {ins.op} needs a .smem declaration")
    if ins.op in ("lds", "sts"):
        return
    if ins.op == "ldg" and prog.buffers[ins.buf] == "wo":
        raise IRError(f"line {ln}: load from write-only buffer {ins.buf}")
    if ins.op in ("stg", "atom.add", "atom.cas") and prog.buffers[ins.buf] == "ro":
        raise IRError(f"line {ln}: write to read-only buffer {ins.buf}")
    if ins.op in ("atom.add", "atom.cas") and prog.buffers[ins.buf] != "rw":
        raise IRError(f"line {ln}: atomics need an rw buffer")
