// Per-pass specialisation of the fused tile kernel (a9) with NVRTC.
//
// The interpreted tile kernel (kernels.cu) walks the pass program op by op; with 16 complex
// amplitudes live in registers the generic dispatch costs more than the arithmetic (register
// moves at the dispatch loop head, predicated code for every possible register bit). Here the
// same device functions (tile_common.cuh) are called in a straight line with the op kinds,
// register-bit indices, matrix classes and r-conditions as compile-time constants; matrices,
// phases and tile-uniform conditions stay run-time data in the pass blob, so one compiled
// kernel serves every circuit with the same pass structure (cache key = generated source).
// NVRTC and the driver API are loaded with dlopen; if unavailable the interpreted kernel runs.
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nvrtc.h>

#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <sstream>
#include <string>
#include <unordered_map>

#include "jit.h"
#include "kernels.h"
#include "qgpu_internal.h"

namespace qgpu {

#include "tile_common_src.inc"  // kTileCommonSrc: tile_common.cuh as a string

namespace {

struct JitLib {
  bool tried = false, ok = false;
  std::string err;
  decltype(&nvrtcCreateProgram) createProgram = nullptr;
  decltype(&nvrtcCompileProgram) compileProgram = nullptr;
  decltype(&nvrtcGetProgramLogSize) getLogSize = nullptr;
  decltype(&nvrtcGetProgramLog) getLog = nullptr;
  decltype(&nvrtcGetCUBINSize) getCubinSize = nullptr;
  decltype(&nvrtcGetCUBIN) getCubin = nullptr;
  decltype(&nvrtcDestroyProgram) destroyProgram = nullptr;
  decltype(&cuModuleLoadData) moduleLoadData = nullptr;
  decltype(&cuModuleGetFunction) moduleGetFunction = nullptr;
  decltype(&cuFuncSetAttribute) funcSetAttribute = nullptr;
  decltype(&cuLaunchKernel) launchKernel = nullptr;
  std::mutex mu;
  std::unordered_map<std::string, CUfunction> cache;
};

JitLib& lib() {
  static JitLib L;
  return L;
}

void* open_first(const char* const* names) {
  for (const char* const* n = names; *n; ++n)
    if (void* h = dlopen(*n, RTLD_NOW | RTLD_GLOBAL)) return h;
  return nullptr;
}

bool load_nvrtc(JitLib& L) {
  static const char* const nv[] = {"libnvrtc.so.12", "/usr/local/cuda/lib64/libnvrtc.so.12", "libnvrtc.so", nullptr};
  void* h = open_first(nv);
  if (!h) {
    L.err = "libnvrtc not found";
    return false;
  }
#define QGPU_SYM(field, name)                                   \
  L.field = reinterpret_cast<decltype(L.field)>(dlsym(h, name)); \
  if (!L.field) {                                               \
    L.err = std::string("missing ") + name;                     \
    return false;                                               \
  }
  QGPU_SYM(createProgram, "nvrtcCreateProgram")
  QGPU_SYM(compileProgram, "nvrtcCompileProgram")
  QGPU_SYM(getLogSize, "nvrtcGetProgramLogSize")
  QGPU_SYM(getLog, "nvrtcGetProgramLog")
  QGPU_SYM(getCubinSize, "nvrtcGetCUBINSize")
  QGPU_SYM(getCubin, "nvrtcGetCUBIN")
  QGPU_SYM(destroyProgram, "nvrtcDestroyProgram")
  return true;
}

bool load_driver(JitLib& L) {
  static const char* const cu[] = {"libcuda.so.1", "libcuda.so", nullptr};
  void* h = open_first(cu);
  if (!h) {
    L.err = "libcuda not found";
    return false;
  }
  QGPU_SYM(moduleLoadData, "cuModuleLoadData")
  QGPU_SYM(moduleGetFunction, "cuModuleGetFunction")
  QGPU_SYM(funcSetAttribute, "cuFuncSetAttribute")
  QGPU_SYM(launchKernel, "cuLaunchKernel")
#undef QGPU_SYM
  return true;
}

}  // namespace

std::string tile_jit_source(const Pass& p) {
  const TileProgram& P = p.prog;
  const int NR = P.nr;
  std::ostringstream o;
  o << "// qgpu tile pass: b=" << p.b << " nr=" << NR << " nw=" << P.nw << " ops=" << P.ops.size() << "\n";
  o << "#include \"tile_common.cuh\"\n";
  o << "using namespace qgpu;\n";
  o << "struct JitBody {\n";
  o << "  __device__ __forceinline__ void operator()(double2 (&v)[kRegAmps], Mapping& mp, const TileCtx& c) const {\n";
  o << "    const TileOp* ops = c.ops;\n";
  for (size_t i = 1; i < P.ops.size(); ++i) {
    const TileOp& op = P.ops[i];
    const bool uni = op.omask != 0;       // tile-uniform condition present
    const bool thr = op.tmask != 0;       // condition on the thread's fixed bits present
    o << "    { const TileOp& op = ops[" << i << "];\n";
    switch (op.kind) {
      case OP_RUN:
        o << "      op_run<" << NR << ">(v, op, c, mp, " << op.a0 << ", " << op.a1 << ", " << op.cls << ", "
          << op.tmask << ", " << op.tmatch << ");\n";
        break;
      case OP_U1R:
        o << "      if (" << (uni ? "op_active(op, c.gbase)" : "true") << (thr ? " && (mp.base & op.tmask) == op.tmatch" : "")
          << ") op_u1r<" << NR << ", " << op.a0 << ", " << op.cls << ">(v, c.pool + op.moff, " << op.rmask << "u, "
          << op.rmatch << "u);\n";
        break;
      case OP_U1L:
        o << "      if (" << (uni ? "op_active(op, c.gbase)" : "true") << ") op_u1l<" << NR << ", " << op.cls
          << ">(v, c.pool + op.moff, " << op.a0 << ", c.lane, " << (thr ? "(mp.base & op.tmask) == op.tmatch" : "true")
          << ", " << op.rmask << "u, " << op.rmatch << "u);\n";
        break;
      case OP_U2R:
        o << "      if (" << (uni ? "op_active(op, c.gbase)" : "true") << (thr ? " && (mp.base & op.tmask) == op.tmatch" : "")
          << ") op_u2r<" << NR << ", " << op.a0 << ", " << op.a1 << ">(v, c.pool + op.moff, " << op.rmask << "u, "
          << op.rmatch << "u);\n";
        break;
      case OP_REMAP:
        o << "      tile_spill<" << NR << ">(v, c, mp); mp = make_mapping<" << NR
          << ">(op, c.nw, c.lane, c.warp); tile_reload<" << NR << ">(v, c, mp);\n";
        break;
      case OP_SMEM1:
      case OP_SMEM2:
        o << "      if (" << (uni ? "op_active(op, c.gbase)" : "true") << ") { tile_spill<" << NR << ">(v, c, mp); ";
        if (op.kind == OP_SMEM2) o << "op_smem2(c, op); ";
        else o << "op_smem1<" << op.cls << ">(c, op); ";
        o << "tile_reload<" << NR << ">(v, c, mp); }\n";
        break;
      default:
        break;
    }
    o << "    }\n";
  }
  o << "  }\n};\n";
  o << "extern \"C\" __global__ void __launch_bounds__(256, 1) qgpu_tile_pass(const TileArgs a) {\n";
  o << "  JitBody body;\n  tile_driver<" << NR << ">(a, body);\n}\n";
  return o.str();
}

bool jit_compile_cubin(const std::string& src, std::string* cubin, std::string* log) {
  JitLib& L = lib();
  if (!L.createProgram && !load_nvrtc(L)) {
    *log = L.err;
    return false;
  }
  nvrtcProgram prog;
  const char* hdrs[] = {kTileCommonSrc};
  const char* names[] = {"tile_common.cuh"};
  if (L.createProgram(&prog, src.c_str(), "qgpu_tile_pass.cu", 1, hdrs, names) != NVRTC_SUCCESS) {
    *log = "nvrtcCreateProgram failed";
    return false;
  }
  const char* opts[] = {"-arch=sm_100a", "-std=c++17", "-lineinfo", "-DQGPU_JIT=1"};
  const nvrtcResult rc = L.compileProgram(prog, 4, opts);
  size_t n = 0;
  L.getLogSize(prog, &n);
  log->assign(n, '\0');
  if (n) L.getLog(prog, &(*log)[0]);
  bool ok = rc == NVRTC_SUCCESS;
  if (ok) {
    size_t cn = 0;
    ok = L.getCubinSize(prog, &cn) == NVRTC_SUCCESS && cn > 0;
    if (ok) {
      cubin->assign(cn, '\0');
      ok = L.getCubin(prog, &(*cubin)[0]) == NVRTC_SUCCESS;
    }
  }
  L.destroyProgram(&prog);
  return ok;
}

bool jit_available(std::string* why) {
  JitLib& L = lib();
  std::lock_guard<std::mutex> g(L.mu);
  if (!L.tried) {
    L.tried = true;
    L.ok = load_nvrtc(L) && load_driver(L);
  }
  if (!L.ok && why) *why = L.err;
  return L.ok;
}

// Compile (or fetch from the cache) and launch the specialised kernel of pass p.
// Returns cudaErrorNotSupported when the JIT is unavailable (caller falls back).
cudaError_t launch_tile_jit(cudaStream_t st, const Pass& p, const TileArgs& a, size_t smem, int num_sms,
                            double* compile_ms) {
  if (!jit_available(nullptr)) return cudaErrorNotSupported;
  JitLib& L = lib();
  const std::string src = tile_jit_source(p);
  CUfunction fn = nullptr;
  {
    std::lock_guard<std::mutex> g(L.mu);
    auto it = L.cache.find(src);
    if (it != L.cache.end()) fn = it->second;
  }
  if (!fn) {
    const auto t0 = std::chrono::steady_clock::now();
    std::string cubin, log;
    if (!jit_compile_cubin(src, &cubin, &log)) {
      std::fprintf(stderr, "qgpu: JIT compile failed, using the interpreted tile kernel:\n%s\n", log.c_str());
      return cudaErrorNotSupported;
    }
    cudaFree(nullptr);  // make sure the runtime's primary context is current for the driver API
    CUmodule mod = nullptr;
    if (L.moduleLoadData(&mod, cubin.data()) != CUDA_SUCCESS) return cudaErrorNotSupported;
    if (L.moduleGetFunction(&fn, mod, "qgpu_tile_pass") != CUDA_SUCCESS) return cudaErrorNotSupported;
    if (L.funcSetAttribute(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, 227 * 1024) != CUDA_SUCCESS)
      return cudaErrorNotSupported;
    const auto t1 = std::chrono::steady_clock::now();
    if (compile_ms) *compile_ms += std::chrono::duration<double, std::milli>(t1 - t0).count();
    std::lock_guard<std::mutex> g(L.mu);
    L.cache.emplace(src, fn);
  }
  const unsigned threads = 32u << a.nw;
  const unsigned grid = unsigned(std::min<uint64_t>(a.ntiles, uint64_t(num_sms)));
  TileArgs args = a;
  void* params[] = {&args};
  const CUresult r = L.launchKernel(fn, grid, 1, 1, threads, 1, 1, unsigned(smem), reinterpret_cast<CUstream>(st),
                                    params, nullptr);
  return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorLaunchFailure;
}

}  // namespace qgpu
