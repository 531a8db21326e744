"""C2s poll overhead at several grid sizes (polled vs no-polls build,
interleaved): the 292-295-block anomaly of profiles/r02_poll_placement.md.
python tools/c2s_overhead_check.py 296,295,288"""
import sys, numpy as np, torch
sys.path.insert(0, '/root/repo')
import bench, paper_conf_ipps_jiw21_b200 as cb
from workloads import configs
cfg = configs.c2s()
dA = torch.from_numpy(cfg["buffers"]["A"].view(np.int32)).cuda()
dB = torch.from_numpy(cfg["buffers"]["B"].view(np.int32)).cuda()
dC = torch.zeros(4096 * 4096, dtype=torch.int32, device="cuda")
mk = lambda: [dA, dB, dC]
for g in [int(x) for x in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["296", "295"])]:
    print(g, bench._poll_overhead(cb, cfg["ir"], g, mk, min_blocks=2))
p = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2)
q = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2, debug=cb.DEBUG_NO_POLLS)
print(p.info['num_regs'], q.info['num_regs'], p.occupancy(), q.occupancy())
