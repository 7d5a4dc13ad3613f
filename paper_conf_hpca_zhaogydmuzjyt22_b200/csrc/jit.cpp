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

#include <algorithm>
#include <bit>
#include <atomic>
#include <chrono>
#include <fstream>
#include <sys/stat.h>
#include <unistd.h>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <thread>
#include <sstream>
#include <string>
#include <unordered_map>
#include <vector>

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
  decltype(&cuOccupancyMaxActiveBlocksPerMultiprocessor) occupancy = nullptr;
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
  QGPU_SYM(occupancy, "cuOccupancyMaxActiveBlocksPerMultiprocessor")
#undef QGPU_SYM
  return true;
}

// ---- on-disk cubin cache: <dir>/<fnv1a64(source|tile_common.cuh|options)>.cubin
// dir = $QGPU_JIT_CACHE, else <directory of libqgpu.so>/build/jitcache
std::string cache_dir() {
  if (const char* ev = std::getenv("QGPU_JIT_CACHE")) return ev;
  Dl_info info;
  if (dladdr(reinterpret_cast<void*>(&cache_dir), &info) && info.dli_fname) {
    std::string so = info.dli_fname;
    const size_t k = so.find_last_of('/');
    return (k == std::string::npos ? std::string(".") : so.substr(0, k)) + "/build/jitcache";
  }
  return "";
}

std::string cache_key(const std::string& src) {
  uint64_t h = 1469598103934665603ull;
  auto mix = [&](const std::string& x) {
    for (unsigned char ch : x) {
      h ^= ch;
      h *= 1099511628211ull;
    }
  };
  mix(src);
  mix(kTileCommonSrc);  // the included device code: a change to it must not hit stale cubins
  mix("|sm_100a|-std=c++17|-lineinfo|");
  if (const char* ev = std::getenv("QGPU_JIT_OPTS")) mix(ev);
  char buf[32];
  std::snprintf(buf, sizeof(buf), "%016llx", static_cast<unsigned long long>(h));
  return buf;
}

bool cache_read(const std::string& key, std::string* cubin) {
  const std::string d = cache_dir();
  if (d.empty()) return false;
  std::ifstream f(d + "/" + key + ".cubin", std::ios::binary);
  if (!f) return false;
  cubin->assign(std::istreambuf_iterator<char>(f), std::istreambuf_iterator<char>());
  return !cubin->empty();
}

void cache_write(const std::string& key, const std::string& cubin) {
  const std::string d = cache_dir();
  if (d.empty()) return;
  ::mkdir((d.substr(0, d.find_last_of('/'))).c_str(), 0755);
  ::mkdir(d.c_str(), 0755);
  const std::string tmp = d + "/" + key + ".tmp." + std::to_string(::getpid());
  {
    std::ofstream f(tmp, std::ios::binary);
    if (!f) return;
    f.write(cubin.data(), std::streamsize(cubin.size()));
  }
  std::rename(tmp.c_str(), (d + "/" + key + ".cubin").c_str());
}

// loaded functions belong to the current device's primary context: the in-memory cache is
// keyed by device ordinal + source (the caller has made the state's device current)
std::string device_tag() {
  int d = 0;
  cudaGetDevice(&d);
  return "dev" + std::to_string(d) + "|";
}

}  // namespace

bool jit_cubin_cached(const std::string& src, std::string* cubin, std::string* log, bool* hit) {
  const std::string key = cache_key(src);
  if (const char* dir = std::getenv("QGPU_JIT_DUMP")) {  // generated sources, for inspection
    std::ofstream f(std::string(dir) + "/qgpu_pass_" + key + ".cu");
    f << src;
  }
  if (cache_read(key, cubin)) {
    if (hit) *hit = true;
    return true;
  }
  if (hit) *hit = false;
  if (!jit_compile_cubin(src, cubin, log)) return false;
  cache_write(key, *cubin);
  return true;
}

std::string tile_jit_source(const Pass& p, int hist_mode, uint32_t hist_key) {
  const bool hist = hist_mode >= 0;
  const TileProgram& P = p.prog;
  const int NR = P.nr;
  // compile-time slot tables of a mapping: tile-local offset J[r] and physical offset Pq[r]
  auto jtab = [&](const int* Rb) {
    std::ostringstream t;
    t << "{";
    for (int r = 0; r < 16; ++r) {
      uint32_t j = 0;
      for (int k = 0; k < NR; ++k)
        if (r >> k & 1) j |= 1u << Rb[k];
      t << (r ? ", " : "") << j << "u";
    }
    t << "}";
    return t.str();
  };
  auto ptab = [&](const int* Rb) {
    std::ostringstream t;
    t << "{";
    for (int r = 0; r < 16; ++r) {
      unsigned long long q = 0;
      for (int k = 0; k < NR; ++k)
        if (r >> k & 1) q |= 1ull << p.spos[Rb[k]];
      t << (r ? ", " : "") << q << "ull";
    }
    t << "}";
    return t.str();
  };
  auto base_expr = [&](const TileOp& op) {
    std::ostringstream t;
    t << "uint32_t(c.lane)";
    for (int k = 0; k < P.nw; ++k)
      t << " | ((c.warp >> " << k << ") & 1 ? " << (1u << ((op.a1 >> (4 * k)) & 15)) << "u : 0u)";
    return t.str();
  };
  // compile-time zero tracking (first-touch expansion, a5): tile bits whose physical position
  // is >= k_in hold zeros until a non-diagonal op targets them
  uint32_t zpos = 0;
  for (int i = 0; i < p.b; ++i)
    if (p.spos[i] >= p.k_in || (p.zin >> p.spos[i] & 1)) zpos |= 1u << i;
  int R[4] = {0, 0, 0, 0};
  auto decode = [&](const TileOp& op) {
    for (int k = 0; k < 4; ++k) R[k] = (op.a0 >> (4 * k)) & 15;
  };
  auto zmask = [&]() {
    unsigned zm = 0;
    for (int r = 0; r < (1 << NR); ++r)
      for (int k = 0; k < NR; ++k)
        if ((r >> k & 1) && (zpos >> R[k] & 1)) zm |= 1u << r;
    return zm;
  };
  uint32_t Wmask = 0;  // tile bits that are warp bits in the current mapping
  int W[4] = {0, 0, 0, 0};  // warp-bit index -> tile bit
  auto decode_w = [&](const TileOp& op) {
    Wmask = 0;
    for (int k = 0; k < P.nw; ++k) {
      W[k] = (op.a1 >> (4 * k)) & 15;
      Wmask |= 1u << W[k];
    }
  };
  // warp-group remaps: (mbarrier base index, number of changed warp-bit indices)
  std::vector<std::pair<int, int>> groups;
  decode(P.ops[0]);
  decode_w(P.ops[0]);
  std::ostringstream o;
  o << "// qgpu tile pass: b=" << p.b << " nr=" << NR << " nw=" << P.nw << " ops=" << P.ops.size()
    << " k_in=" << p.k_in << "\n";
  o << "#include \"tile_common.cuh\"\n";
  o << "using namespace qgpu;\n";
  // zero slots / zero warps at the start of the pass (used by the driver to skip loads)
  const unsigned zm_start = zmask();
  const uint32_t zw_start = zpos & Wmask;
  // final mapping (for the store)
  int RF[4] = {R[0], R[1], R[2], R[3]};
  for (const TileOp& op : P.ops)
    if (op.kind == OP_REMAP)
      for (int k = 0; k < 4; ++k) RF[k] = (op.a0 >> (4 * k)) & 15;
  std::ostringstream body, hdr;
  bool fold_scalar = false;  // the tile-uniform scalar joins the first run (see below)
  {
    std::ostringstream& o = body;  // the program body is generated first (it fixes the barriers)
  hdr << "  static constexpr unsigned kZM0 = " << zm_start << "u;\n";
  hdr << "  static constexpr uint32_t kZW0 = " << zw_start << "u;\n";
  hdr << "  static constexpr bool kStatic = true;\n";
  hdr << "  static constexpr bool kHist = " << (hist ? "true" : "false") << ";\n";
  hdr << "  static constexpr int kHistMode = " << (hist ? hist_mode : 0) << ";\n";
  {
    const bool rs = hist && hist_mode == 2 && hist_key != ~0u;
    hdr << "  static constexpr bool kHistRS = " << (rs ? "true" : "false") << ";\n";
    hdr << "  static constexpr uint32_t kHlred = " << (rs ? (hist_key & 0xffu) : 0u) << "u;\n";
    hdr << "  static constexpr uint32_t kDead = " << (rs ? (hist_key >> 8 & 0xfu) : 0u) << "u;\n";
    hdr << "  static constexpr bool kHistGlob = " << (rs && (hist_key >> 12 & 1u) ? "true" : "false") << ";\n";
  }
  {  // tile positions as runs of consecutive bits (tile index -> base address at compile time)
    std::vector<int> rp, rl;
    for (int i = 0; i < p.b;) {
      int j = i;
      while (j + 1 < p.b && p.spos[j + 1] == p.spos[j] + 1) ++j;
      rp.push_back(p.spos[i]);
      rl.push_back(j - i + 1);
      i = j + 1;
    }
    auto arr = [](const std::vector<int>& v) {
      std::string t = "{";
      for (size_t i = 0; i < v.size(); ++i) t += (i ? ", " : "") + std::to_string(v[i]);
      return t + "}";
    };
    hdr << "  static constexpr int kNsrun = " << rp.size() << ";\n";
    hdr << "  static constexpr int kSrunPos[" << rp.size() << "] = " << arr(rp) << ";\n";
    hdr << "  static constexpr int kSrunLen[" << rl.size() << "] = " << arr(rl) << ";\n";
  }
  hdr << "  static constexpr bool kHasScalar = " << (P.scalar.empty() ? "false" : "true") << ";\n";
  hdr << "  static constexpr uint32_t kJ0[kRegAmps] = " << jtab(R) << ";\n";
  hdr << "  static constexpr uint64_t kP0[kRegAmps] = " << ptab(R) << ";\n";
  hdr << "  static constexpr uint64_t kPF[kRegAmps] = " << ptab(RF) << ";\n";
  hdr << "  static constexpr uint32_t kJF[kRegAmps] = " << jtab(RF) << ";\n";
  // the last op that touches the tile buffer (remap, shared-memory op): after it the program
  // runs from registers, so the driver's prefetch of the next tile into the single buffer of a
  // two-CTA pass can be issued there (pf) instead of after the whole program
  size_t last_smem = 0;
  for (size_t i = 1; i < P.ops.size(); ++i)
    if (P.ops[i].kind == OP_REMAP || P.ops[i].kind == OP_SMEM1 || P.ops[i].kind == OP_SMEM2) last_smem = i;
  // only for programs with at most two remaps and >= 3 compute ops after the last one (A/B,
  // profiles/r02b: QAOA_32, one or two remaps mid-program, 49.0 -> 48.0 ms; rqc_30, many remaps,
  // 111.2 -> 112.2 ms with it on every pass, also when gated on the ops after the last remap only)
  {
    int after = 0, nremap = 0;
    for (size_t i = 1; i < P.ops.size(); ++i) nremap += P.ops[i].kind == OP_REMAP;
    for (size_t i = last_smem + 1; i < P.ops.size() && last_smem > 0; ++i)
      after += (P.ops[i].kind == OP_RUN || P.ops[i].kind == OP_U1R || P.ops[i].kind == OP_U1L ||
                P.ops[i].kind == OP_U2R);
    const char* ev = std::getenv("QGPU_EARLY_PF");  // 0: after the program, 1: gated, 2: always
    const int mode = ev ? std::atoi(ev) : 0;  // default off since the scalar folding (r3o: 46.0
                                               // vs 46.7 ms with it on QAOA_32, one-table runs)
    if (mode == 0 || (mode == 1 && (after < 3 || nremap > 2))) last_smem = 0;
  }
  hdr << "  static constexpr bool kEarlyPrefetch = " << (last_smem > 0 ? "true" : "false") << ";\n";
  o << "  template <class PF>\n";
  o << "  __device__ __forceinline__ void operator()(double2 (&v)[kRegAmps], Mapping& mp, const TileCtx& c, const TileArgs& a, PF&& pf) const {\n";
  o << "    const TileOp* ops = c.ops;\n";
  {
    const unsigned zm = zmask();
    if (zm) {  // the initial reload read these slots from the zero region: make them exact zeros
      o << "    {";
      for (int r = 0; r < (1 << NR); ++r)
        if (zm >> r & 1) o << " v[" << r << "] = make_double2(0.0, 0.0);";
      o << " }\n";
    }
  }
  // U matrices: from the kernel-parameter pool at compile-time offsets when the pool fits
  // (TileArgs::umat), else from the program blob in shared memory
  const bool upar = P.pool.size() <= size_t(kUmatParam);
  auto umat = [&](const TileOp& op) {
    return upar ? "a.umat + " + std::to_string(op.moff) : std::string("c.pool + op.moff");
  };
  // conditions as compile-time constants (they are structural: positions, not values)
  auto active = [&](const TileOp& op) {
    std::ostringstream t;
    t << "((c.gbase & " << op.omask << "ull) == " << op.omatch << "ull)";
    return t.str();
  };
  auto thrc = [&](const TileOp& op) {
    std::ostringstream t;
    t << "((mp.base & " << op.tmask << "u) == " << op.tmatch << "u)";
    return t.str();
  };
  // the tile-uniform scalar (phase terms on bits outside the tile and the deferred factors of
  // the unit-diagonal matrix forms) commutes with the whole program: it joins the first run's
  // t0 (every owned non-zero amplitude passes through it; by linearity the amplitudes that are
  // still zero there carry it once they are formed) instead of a separate multiply of every
  // amplitude at the end of the tile (QGPU_FOLD_SCALAR=0: A/B)
  fold_scalar = !P.scalar.empty() && P.spat >= 0;
  if (const char* ev = std::getenv("QGPU_FOLD_SCALAR"))
    if (std::atoi(ev) == 0) fold_scalar = false;
  {
    bool has_run = false;
    for (size_t i = 1; i < P.ops.size(); ++i) has_run = has_run || P.ops[i].kind == OP_RUN;
    fold_scalar = fold_scalar && has_run;
  }
  bool scalar_pending = fold_scalar;
  for (size_t i = 1; i < P.ops.size(); ++i) {
    const TileOp& op = P.ops[i];
    const bool uni = op.omask != 0;       // tile-uniform condition present
    const bool thr = op.tmask != 0;       // condition on the thread's fixed bits present
    const unsigned zm = zmask();
    const uint32_t zw = zpos & Wmask;  // warps whose fixed bits hit these hold only zeros
    o << "    { const TileOp& op = ops[" << i << "];\n";
    const bool wguard = zw && (op.kind == OP_RUN || op.kind == OP_U1R || op.kind == OP_U2R || op.kind == OP_U1L);
    if (wguard) o << "      if ((mp.base & " << zw << "u) == 0u) {\n";
    switch (op.kind) {
      case OP_RUN: {
        // entries are compile-time: slot 0 (all owned amplitudes), slots 1..4 (r bit k set),
        // then general groups (compile-time r condition); zero slots are skipped
        const int ns[5] = {op.a0, op.a1, op.cls, int(op.tmask), int(op.tmatch)};
        const char* acc[5] = {"t0", "e0", "e1", "e2", "e3"};
        uint32_t e = op.moff;
        o << "      const uint32_t tb = mp.base; (void)tb;\n";
        o << "      const double2 one = make_double2(1.0, 0.0); (void)one;\n";
        // the product of a list of entries: entries with equal tmask have distinct tmatch, so at
        // most one of them matches a thread -> one select per tmask group, one cmul per extra
        // group, and an unconditional entry is a plain load
        auto product = [&](const char* name, uint32_t e0, uint32_t e1) {
          std::vector<uint32_t> masks;
          for (uint32_t q = e0; q < e1; ++q)
            if (std::find(masks.begin(), masks.end(), P.entries[q].tmask) == masks.end())
              masks.push_back(P.entries[q].tmask);
          for (size_t gi = 0; gi < masks.size(); ++gi) {
            const uint32_t m = masks[gi];
            const std::string f = gi == 0 ? std::string(name) : std::string("f");
            o << "      { double2 f;\n" + std::string(gi == 0 ? "" : "");
            if (m == 0) {
              for (uint32_t q = e0; q < e1; ++q)
                if (P.entries[q].tmask == 0) o << "        f = c.C[" << P.entries[q].pat << "];\n";
            } else {
              o << "        f = one;\n";
              for (uint32_t q = e0; q < e1; ++q)
                if (P.entries[q].tmask == m)
                  o << "        if ((tb & " << m << "u) == " << P.entries[q].tmatch << "u) f = c.C["
                    << P.entries[q].pat << "];\n";
            }
            if (gi == 0) o << "        " << name << " = f; }\n";
            else o << "        " << name << " = cmul(" << name << ", f); }\n";
            (void)f;
          }
        };
        o << "      double2 t0 = one, e0 = one, e1 = one, e2 = one, e3 = one;\n";
        int used = 0;
        for (int sl = 0; sl < 5; ++sl) {
          if (ns[sl]) used |= 1 << sl;
          product(acc[sl], e, e + uint32_t(ns[sl]));
          e += uint32_t(ns[sl]);
        }
        if (scalar_pending) {
          o << "      t0 = cmul(t0, c.C[" << P.spat << "]);  // the tile-uniform scalar\n";
          used |= 1;
          scalar_pending = false;
        }
        // general groups (compile-time r condition). Phase factors have modulus 1, so a factor
        // a on "r bit k clear" is a on all slots times conj(a) on "r bit k set" (two doubling
        // factors of the P-table instead of 8 multiplies), and a pair a on (r_i, r_j) = (1, 0),
        // b on (0, 1) is e_i *= a, e_j *= b and conj(a b) on (1, 1) (4 multiplies instead of 8)
        struct Grp {
          uint32_t g0, g1, rm, rt;
          bool done;
        };
        std::vector<Grp> grps;
        const uint32_t end = op.moff + op.cnt;
        for (uint32_t g0 = e; g0 < end;) {
          uint32_t g1 = g0;
          while (!P.entries[g1].gend) ++g1;
          grps.push_back({g0, g1 + 1, P.entries[g0].rmask, P.entries[g0].rmatch, false});
          g0 = g1 + 1;
        }
        std::vector<std::pair<uint32_t, std::string>> late;  // (r mask, factor) applied on r & mask == mask
        int nfac = 0;
        for (Grp& g : grps) {
          if (std::popcount(g.rm) == 1 && g.rt == 0) {
            const int k = std::countr_zero(g.rm);
            o << "      { double2 acc;\n";
            product("acc", g.g0, g.g1);
            o << "        t0 = cmul(t0, acc); " << acc[1 + k] << " = cmul(" << acc[1 + k]
              << ", make_double2(acc.x, -acc.y)); }\n";
            used |= 1 | (2 << k);
            g.done = true;
          }
        }
        for (size_t x = 0; x < grps.size(); ++x) {
          Grp& A = grps[x];
          if (A.done || std::popcount(A.rm) != 2 || std::popcount(A.rt) != 1) continue;
          for (size_t y = x + 1; y < grps.size(); ++y) {
            Grp& B = grps[y];
            if (B.done || B.rm != A.rm || B.rt != (A.rm & ~A.rt)) continue;
            const int i = std::countr_zero(A.rt), j = std::countr_zero(B.rt);
            const std::string fn = "fac" + std::to_string(nfac++);
            o << "      double2 " << fn << ";\n      { double2 fa, fb;\n";
            product("fa", A.g0, A.g1);
            product("fb", B.g0, B.g1);
            o << "        " << acc[1 + i] << " = cmul(" << acc[1 + i] << ", fa); " << acc[1 + j] << " = cmul("
              << acc[1 + j] << ", fb);\n        " << fn << " = cmul(fa, fb); " << fn << ".y = -" << fn << ".y; }\n";
            used |= (2 << i) | (2 << j);
            late.push_back({A.rm, fn});
            A.done = B.done = true;
            break;
          }
        }
        // one 16-entry factor table (run_apply_ptab_z); QGPU_RUN_SPLIT=1: two 4-entry tables
        // (fewer live registers; measured slower once the scalar was folded into the first run:
        // profiles/r02b ab r3o, QAOA_32 46.8 -> 46.0 ms, rqc_30 96.4 -> 93.6 ms with one table)
        const char* rs_env = std::getenv("QGPU_RUN_SPLIT");
        const bool split_tab = NR == 4 && (rs_env && rs_env[0] == '1');
        if (used)
          o << "      " << (split_tab ? "run_apply_split_z<" : "run_apply_ptab_z<") << NR << ", " << (used & 1 ? "true" : "false") << ", "
            << ((used >> 1) & 1 ? "true" : "false") << ", " << ((used >> 2) & 1 ? "true" : "false") << ", "
            << ((used >> 3) & 1 ? "true" : "false") << ", " << ((used >> 4) & 1 ? "true" : "false") << ", " << zm
            << "u>(v, t0, e0, e1, e2, e3);\n";
        for (const auto& lf : late)
          o << "      run_apply_group_z<" << NR << ", " << lf.first << "u, " << lf.first << "u, " << zm << "u>(v, "
            << lf.second << ");\n";
        for (const Grp& g : grps) {
          if (g.done) continue;
          o << "      { double2 acc;\n";
          product("acc", g.g0, g.g1);
          o << "        run_apply_group_z<" << NR << ", " << g.rm << "u, " << g.rt << "u, " << zm << "u>(v, acc); }\n";
        }
        break;
      }
      case OP_U1R:
        o << "      if (" << (uni ? active(op) : "true") << (thr ? " && " + thrc(op) : "")
          << ") op_u1r_z<" << NR << ", " << op.a0 << ", " << op.cls << ", " << zm << "u>(v, " << umat(op) << ", "
          << op.rmask << "u, " << op.rmatch << "u);\n";
        zpos &= ~(1u << R[op.a0]);
        break;
      case OP_U1L:
        o << "      if (" << (uni ? active(op) : "true") << ") op_u1l_z<" << NR << ", " << op.cls
          << ", " << zm << "u>(v, " << umat(op) << ", " << op.a0 << ", c.lane, "
          << (thr ? thrc(op) : "true") << ", " << op.rmask << "u, " << op.rmatch << "u);\n";
        zpos &= ~(1u << op.a0);
        break;
      case OP_U2R:
        o << "      if (" << (uni ? active(op) : "true") << (thr ? " && " + thrc(op) : "")
          << ") op_u2r_z<" << NR << ", " << op.a0 << ", " << op.a1 << ", " << zm << "u>(v, " << umat(op) << ", "
          << op.rmask << "u, " << op.rmatch << "u);\n";
        zpos &= ~((1u << R[op.a0]) | (1u << R[op.a1]));
        break;
      case OP_REMAP: {
        int Wold[4] = {W[0], W[1], W[2], W[3]};
        o << "      { constexpr uint32_t Jo[kRegAmps] = " << jtab(R) << ";\n";
        o << "        tile_store_j<" << NR << ">(v, c, mp.base, Jo); }\n";
        decode(op);
        decode_w(op);
        {
          int nchg = 0;
          std::string gexpr = "0";
          int gi = 0;
          for (int k = 0; k < P.nw; ++k) {
            if (W[k] != Wold[k]) {
              ++nchg;
            } else {
              gexpr += " | (((c.warp >> " + std::to_string(k) + ") & 1) << " + std::to_string(gi) + ")";
              ++gi;
            }
          }
          if (nchg > 0) {  // nchg == 0: the thread's own slots, a register permutation
            const int base = int(groups.size()) << P.nw;
            groups.push_back({base, nchg});
            o << "      group_sync(c, " << base << " + (" << gexpr << "));\n";
          }
        }
        o << "      mp.base = " << base_expr(op) << ";\n";
        o << "      { constexpr uint32_t Jn[kRegAmps] = " << jtab(R) << ";\n";
        o << "        tile_reload_j<" << NR << ">(v, c, mp.base, Jn); }\n";
        break;
      }
      case OP_SMEM1:
      case OP_SMEM2:
        o << "      if (" << (uni ? active(op) : "true") << ") { constexpr uint32_t Jc[kRegAmps] = "
          << jtab(R) << ";\n        tile_spill_j<" << NR << ">(v, c, mp.base, Jc); ";
        if (op.kind == OP_SMEM2) o << "op_smem2(c, op); ";
        else o << "op_smem1<" << op.cls << ">(c, op); ";
        o << "tile_reload_j<" << NR << ">(v, c, mp.base, Jc); }\n";
        zpos &= ~(1u << op.a0);
        if (op.kind == OP_SMEM2) zpos &= ~(1u << op.a1);
        break;
      default:
        break;
    }
    if (wguard) o << "      }\n";
    o << "    }\n";
    if (i == last_smem) o << "    pf();  // the tile buffer is free from here on\n";
  }
  o << "  }\n";
  }
  o << "struct JitBody {\n" << hdr.str();
  o << "  static constexpr bool kScalarFolded = " << (fold_scalar ? "true" : "false") << ";\n";
  o << "  static constexpr bool kGroupRemap = true;\n";
  o << "  __device__ static void init_mbar(uint64_t* mb) {\n";
  for (const auto& g : groups)
    for (int q = 0; q < (1 << (P.nw - g.second)); ++q)
      o << "    mbar_init(mb + " << (g.first + q) << ", " << (32 << g.second) << "u);\n";
  o << "  }\n";
  o << body.str() << "};\n";
  // one CTA per SM with up to 255 registers: measured faster than 2 CTAs/SM at <= 128
  // registers even for the single-buffer (remap-free) programs
  int minb = pass_two_cta(p) ? 2 : 1;  // CTAs per SM the register budget is cut for
  if (const char* ev = std::getenv("QGPU_JIT_MINBLOCKS")) minb = std::max(1, std::atoi(ev));
  o << "extern \"C\" __global__ void __launch_bounds__(" << (NR >= 4 ? 256 : 512) << ", " << minb
    << ") qgpu_tile_pass(const TileArgs a) {\n";
  o << "  JitBody body;\n  tile_driver<" << NR << ">(a, body);\n}\n";
  return o.str();
}

bool jit_compile_cubin(const std::string& src, std::string* cubin, std::string* log) {  // NOLINT
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
  std::vector<const char*> opts = {"-arch=sm_100a", "-std=c++17", "-lineinfo", "-DQGPU_JIT=1"};
  std::vector<std::string> extra;
  if (const char* ev = std::getenv("QGPU_JIT_OPTS")) {  // e.g. "-Xptxas -O2" (experiments)
    std::istringstream is(ev);
    for (std::string w; is >> w;) extra.push_back(w);
  }
  for (auto& w : extra) opts.push_back(w.c_str());
  const nvrtcResult rc = L.compileProgram(prog, int(opts.size()), opts.data());
  size_t n = 0;
  L.getLogSize(prog, &n);
  log->assign(n, '\0');
  if (n) L.getLog(prog, &(*log)[0]);
  if (std::getenv("QGPU_JIT_LOG") && n > 1) std::fprintf(stderr, "qgpu: NVRTC log:\n%s\n", log->c_str());
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

// Make sure the kernels of `passes` are loaded: cubins come from the disk cache or are compiled
// in parallel (one NVRTC program per pass, up to hardware_concurrency threads).
int jit_prepare(const std::vector<const Pass*>& passes, double* compile_ms) {
  if (passes.empty() || !jit_available(nullptr)) return 0;
  JitLib& L = lib();
  const auto t0 = std::chrono::steady_clock::now();
  std::vector<std::string> srcs;
  const std::string dev = device_tag();
  {
    std::lock_guard<std::mutex> g(L.mu);
    for (const Pass* p : passes) {
      std::string src = tile_jit_source(*p);
      if (!L.cache.count(dev + src) && std::find(srcs.begin(), srcs.end(), src) == srcs.end()) srcs.push_back(std::move(src));
    }
  }
  if (srcs.empty()) return 0;
  std::vector<std::string> cubins(srcs.size());
  std::vector<char> ok(srcs.size(), 0);
  std::atomic<size_t> next{0};
  auto work = [&]() {
    for (size_t i; (i = next.fetch_add(1)) < srcs.size();) {
      std::string log;
      ok[i] = jit_cubin_cached(srcs[i], &cubins[i], &log, nullptr) ? 1 : 0;
      if (!ok[i]) std::fprintf(stderr, "qgpu: JIT compile failed:\n%s\n", log.c_str());
    }
  };
  const unsigned nt = std::max(1u, std::min<unsigned>(std::thread::hardware_concurrency(), unsigned(srcs.size())));
  std::vector<std::thread> th;
  for (unsigned t = 1; t < nt; ++t) th.emplace_back(work);
  work();
  for (auto& t : th) t.join();
  cudaFree(nullptr);
  int loaded = 0;
  for (size_t i = 0; i < srcs.size(); ++i) {
    if (!ok[i]) continue;
    CUmodule mod = nullptr;
    CUfunction fn = nullptr;
    if (L.moduleLoadData(&mod, cubins[i].data()) != CUDA_SUCCESS) continue;
    if (L.moduleGetFunction(&fn, mod, "qgpu_tile_pass") != CUDA_SUCCESS) continue;
    if (L.funcSetAttribute(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, 227 * 1024) != CUDA_SUCCESS) continue;
    std::lock_guard<std::mutex> g(L.mu);
    L.cache.emplace(dev + srcs[i], fn);
    ++loaded;
  }
  if (compile_ms)
    *compile_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return loaded;
}

// Compile-time masks of the mode-2 measurement epilogue: the unrequested lane bits (a.hlred,
// low 8 bits) and the register bits of the pass's final mapping whose positions are not
// requested ("dead": their slots share buckets, bits 8..11), bit 12 = a.hglob
uint32_t hist_rs_key(const Pass& p, const TileArgs& a) {
  const TileProgram& P = p.prog;
  int RF[4] = {0, 0, 0, 0};
  for (const TileOp& op : P.ops)
    if (op.kind == OP_REMAP)
      for (int k = 0; k < 4; ++k) RF[k] = (op.a0 >> (4 * k)) & 15;
  uint32_t dead = 0;
  for (int k = 0; k < P.nr; ++k) {
    const int pos = p.spos[RF[k]];
    bool req = false;
    for (int j = 0; j < a.hm; ++j) req = req || a.hpos[j] == pos;
    if (!req) dead |= 1u << k;
  }
  return (a.hlred & 0xffu) | (dead << 8) | (a.hglob ? 1u << 12 : 0u);
}

// Compile (or fetch from the cache) and launch the specialised kernel of pass p.
// Returns cudaErrorNotSupported when the JIT is unavailable (caller falls back).
cudaError_t launch_tile_jit(cudaStream_t st, const Pass& p, const TileArgs& a, size_t smem, int num_sms,
                            double* compile_ms) {
  if (!jit_available(nullptr)) return cudaErrorNotSupported;
  JitLib& L = lib();
  const bool hist = a.hist != nullptr;  // fused measurement: its own variant
  const int hmode = hist ? std::clamp(a.hacc, 0, 2) : -1;
  const uint32_t hkey = hmode == 2 ? hist_rs_key(p, a) : ~0u;
  CUfunction fn = static_cast<CUfunction>(hist ? p.jit_fn_hist[hmode] : p.jit_fn);
  if (hmode == 2 && p.jit_hist_key != hkey) fn = nullptr;  // another measured-qubit set
  std::string src;
  const std::string dev = device_tag();
  if (!fn) {
    src = tile_jit_source(p, hmode, hkey);
    std::lock_guard<std::mutex> g(L.mu);
    auto it = L.cache.find(dev + src);
    if (it != L.cache.end()) fn = it->second;
  }
  if (!fn) {
    const auto t0 = std::chrono::steady_clock::now();
    std::string cubin, log;
    bool hit = false;
    if (!jit_cubin_cached(src, &cubin, &log, &hit)) {
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
    if (compile_ms) *compile_ms += std::max(1e-3, std::chrono::duration<double, std::milli>(t1 - t0).count());
    std::lock_guard<std::mutex> g(L.mu);
    L.cache.emplace(dev + src, fn);
  }
  (hist ? p.jit_fn_hist[hmode] : p.jit_fn) = fn;  // later launches skip source generation and lookup
  if (hmode == 2) p.jit_hist_key = hkey;
  const unsigned threads = 32u << a.nw;
  int bps = 1;
  if (L.occupancy(&bps, fn, int(threads), smem) != CUDA_SUCCESS || bps < 1) bps = 1;
  const unsigned grid = unsigned(std::min<uint64_t>(a.ntiles, uint64_t(num_sms) * uint64_t(bps)));
  TileArgs args = a;
  void* params[] = {&args};
  const CUresult r = L.launchKernel(fn, grid, 1, 1, threads, 1, 1, unsigned(smem), reinterpret_cast<CUstream>(st),
                                    params, nullptr);
  return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorLaunchFailure;
}

}  // namespace qgpu
