#include "driver.h"

#include <dlfcn.h>

#include <mutex>

namespace ctxb {
namespace {

template <class F>
bool sym(void* h, const char* name, F* out, std::string* err) {
  void* p = dlsym(h, name);
  if (!p) {
    *err = std::string("missing symbol ") + name;
    return false;
  }
  *out = reinterpret_cast<F>(p);
  return true;
}

}  // namespace

Driver& driver() {
  static Driver d;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
      d.err = std::string("cannot load the CUDA driver (libcuda.so.1): ") + dlerror();
      return;
    }
    std::string& e = d.err;
    bool ok = sym(h, "cuInit", &d.cuInit, &e) && sym(h, "cuDeviceGet", &d.cuDeviceGet, &e) &&
              sym(h, "cuDevicePrimaryCtxRetain", &d.cuDevicePrimaryCtxRetain, &e) &&
              sym(h, "cuCtxGetCurrent", &d.cuCtxGetCurrent, &e) && sym(h, "cuCtxSetCurrent", &d.cuCtxSetCurrent, &e) &&
              sym(h, "cuCtxGetDevice", &d.cuCtxGetDevice, &e) &&
              sym(h, "cuDeviceGetAttribute", &d.cuDeviceGetAttribute, &e) &&
              sym(h, "cuModuleLoadData", &d.cuModuleLoadData, &e) && sym(h, "cuModuleUnload", &d.cuModuleUnload, &e) &&
              sym(h, "cuModuleGetFunction", &d.cuModuleGetFunction, &e) &&
              sym(h, "cuFuncGetAttribute", &d.cuFuncGetAttribute, &e) &&
              sym(h, "cuFuncSetAttribute", &d.cuFuncSetAttribute, &e) &&
              sym(h, "cuOccupancyMaxActiveBlocksPerMultiprocessor", &d.cuOccupancyMaxActiveBlocksPerMultiprocessor, &e) &&
              sym(h, "cuLaunchKernel", &d.cuLaunchKernel, &e) && sym(h, "cuMemAlloc_v2", &d.cuMemAlloc, &e) &&
              sym(h, "cuMemFree_v2", &d.cuMemFree, &e) && sym(h, "cuMemcpyHtoD_v2", &d.cuMemcpyHtoD, &e) &&
              sym(h, "cuMemcpyDtoH_v2", &d.cuMemcpyDtoH, &e) &&
              sym(h, "cuMemcpyHtoDAsync_v2", &d.cuMemcpyHtoDAsync, &e) &&
              sym(h, "cuMemsetD32Async", &d.cuMemsetD32Async, &e) && sym(h, "cuMemsetD8Async", &d.cuMemsetD8Async, &e) &&
              sym(h, "cuStreamSynchronize", &d.cuStreamSynchronize, &e) &&
              sym(h, "cuGetErrorString", &d.cuGetErrorString, &e) &&
              sym(h, "cuEventCreate", &d.cuEventCreate, &e) && sym(h, "cuEventRecord", &d.cuEventRecord, &e) &&
              sym(h, "cuEventSynchronize", &d.cuEventSynchronize, &e) &&
              sym(h, "cuEventElapsedTime", &d.cuEventElapsedTime, &e) &&
              sym(h, "cuEventDestroy_v2", &d.cuEventDestroy, &e) && sym(h, "cuEventQuery", &d.cuEventQuery, &e) &&
              sym(h, "cuStreamCreate", &d.cuStreamCreate, &e) && sym(h, "cuStreamDestroy_v2", &d.cuStreamDestroy, &e) &&
              sym(h, "cuMemcpyDtoHAsync_v2", &d.cuMemcpyDtoHAsync, &e) &&
              sym(h, "cuMemHostAlloc", &d.cuMemHostAlloc, &e) && sym(h, "cuMemFreeHost", &d.cuMemFreeHost, &e) &&
              sym(h, "cuMemHostGetDevicePointer_v2", &d.cuMemHostGetDevicePointer, &e) &&
              sym(h, "cuStreamCreateWithPriority", &d.cuStreamCreateWithPriority, &e) &&
              sym(h, "cuCtxGetStreamPriorityRange", &d.cuCtxGetStreamPriorityRange, &e) &&
              sym(h, "cuStreamWaitEvent", &d.cuStreamWaitEvent, &e) &&
              sym(h, "cuStreamGetFlags", &d.cuStreamGetFlags, &e);
    if (ok && !sym(h, "cuStreamWriteValue32_v2", &d.cuStreamWriteValue32, &e))
      ok = sym(h, "cuStreamWriteValue32", &d.cuStreamWriteValue32, &e);
    if (ok && !sym(h, "cuStreamBatchMemOp_v2", &d.cuStreamBatchMemOp, &e))
      ok = sym(h, "cuStreamBatchMemOp", &d.cuStreamBatchMemOp, &e);
    if (ok && !sym(h, "cuStreamWaitValue32_v2", &d.cuStreamWaitValue32, &e))
      ok = sym(h, "cuStreamWaitValue32", &d.cuStreamWaitValue32, &e);
    if (!ok) return;
    CUresult r = d.cuInit(0);
    if (r != CUDA_SUCCESS) {
      const char* s = nullptr;
      d.cuGetErrorString(r, &s);
      d.err = std::string("cuInit failed: ") + (s ? s : "?");
      return;
    }
    d.ok = true;
  });
  return d;
}

Nvrtc& nvrtc() {
  static Nvrtc n;
  static std::once_flag once;
  std::call_once(once, [] {
    // NVRTC dlopen()s its builtins library by soname; preload it from the
    // toolkit so no LD_LIBRARY_PATH is needed.
    const char* dirs[] = {"/usr/local/cuda/lib64/", "/usr/local/cuda/targets/x86_64-linux/lib/", ""};
    void* h = nullptr;
    for (const char* dir : dirs) {
      std::string b = std::string(dir) + "libnvrtc-builtins.so.12.9";
      dlopen(b.c_str(), RTLD_NOW | RTLD_GLOBAL);
      std::string p = std::string(dir) + "libnvrtc.so.12";
      h = dlopen(p.c_str(), RTLD_NOW | RTLD_GLOBAL);
      if (h) break;
    }
    if (!h) {
      n.err = std::string("cannot load NVRTC (libnvrtc.so.12): ") + dlerror();
      return;
    }
    std::string& e = n.err;
    n.ok = sym(h, "nvrtcCreateProgram", &n.CreateProgram, &e) && sym(h, "nvrtcCompileProgram", &n.CompileProgram, &e) &&
           sym(h, "nvrtcGetProgramLogSize", &n.GetProgramLogSize, &e) &&
           sym(h, "nvrtcGetProgramLog", &n.GetProgramLog, &e) && sym(h, "nvrtcGetCUBINSize", &n.GetCUBINSize, &e) &&
           sym(h, "nvrtcGetCUBIN", &n.GetCUBIN, &e) && sym(h, "nvrtcDestroyProgram", &n.DestroyProgram, &e) &&
           sym(h, "nvrtcGetErrorString", &n.GetErrorString, &e);
  });
  return n;
}

}  // namespace ctxb
