// jit.cpp — plan-specialised builds of the fused pipeline kernel.
//
// The kernel body (pipeline_body.cuh) reads its plan shape through `K`. Here
// the shape of a lowered plan (every count, kind, width, offset and constant
// of PipeDesc except run-time pointers and sizes) is printed as a constexpr
// descriptor, the same body is compiled by NVRTC for sm_100a with that
// descriptor, and the cubin is loaded with the runtime library API. Result:
// one straight-line kernel per plan with all operator loops unrolled and all
// constants folded — the query-compilation analogue of the paper's per-query
// kernel configuration, done once per distinct plan shape and
// cached for the life of the process.
//
// NVRTC is loaded lazily with dlopen (libnvrtc.so.12); without it the
// precompiled generic kernel runs (same body, shape read at run time).
#include <dlfcn.h>

#include <climits>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

#include "kernels.h"

namespace gpl {

extern const char* const kJitSourceNames[];
extern const char* const kJitSources[];
extern const int kJitNumSources;

namespace {

typedef int nvrtcResult;
typedef struct _nvrtcProgram* nvrtcProgram;

struct Nvrtc {
  bool ok = false;
  std::string why;
  nvrtcResult (*create)(nvrtcProgram*, const char*, const char*, int, const char* const*, const char* const*) = nullptr;
  nvrtcResult (*compile)(nvrtcProgram, int, const char* const*) = nullptr;
  nvrtcResult (*log_size)(nvrtcProgram, size_t*) = nullptr;
  nvrtcResult (*log)(nvrtcProgram, char*) = nullptr;
  nvrtcResult (*cubin_size)(nvrtcProgram, size_t*) = nullptr;
  nvrtcResult (*cubin)(nvrtcProgram, char*) = nullptr;
  nvrtcResult (*destroy)(nvrtcProgram*) = nullptr;
};

Nvrtc load_nvrtc() {
  Nvrtc n;
  const char* names[] = {"libnvrtc.so.12", "libnvrtc.so", "/usr/local/cuda/lib64/libnvrtc.so.12"};
  void* h = nullptr;
  for (const char* nm : names)
    if ((h = dlopen(nm, RTLD_NOW | RTLD_LOCAL))) break;
  if (!h) {
    n.why = "libnvrtc.so.12 not found";
    return n;
  }
  auto sym = [&](const char* s) { return dlsym(h, s); };
  n.create = (decltype(n.create))sym("nvrtcCreateProgram");
  n.compile = (decltype(n.compile))sym("nvrtcCompileProgram");
  n.log_size = (decltype(n.log_size))sym("nvrtcGetProgramLogSize");
  n.log = (decltype(n.log))sym("nvrtcGetProgramLog");
  n.cubin_size = (decltype(n.cubin_size))sym("nvrtcGetCUBINSize");
  n.cubin = (decltype(n.cubin))sym("nvrtcGetCUBIN");
  n.destroy = (decltype(n.destroy))sym("nvrtcDestroyProgram");
  n.ok = n.create && n.compile && n.log_size && n.log && n.cubin_size && n.cubin && n.destroy;
  if (!n.ok) n.why = "libnvrtc lacks a required symbol";
  return n;
}

Nvrtc& nvrtc() {
  static Nvrtc n = load_nvrtc();
  return n;
}

struct Entry {
  std::vector<char> cubin;
  cudaLibrary_t lib = nullptr;
  cudaKernel_t kernel = nullptr;
  std::string err;
};
std::mutex g_mu;
std::map<std::string, Entry> g_cache;

std::string i64(long long v) {
  if (v == LLONG_MIN) return "(-9223372036854775807LL - 1)";
  return std::to_string(v) + "LL";
}
std::string u64(unsigned long long v) { return std::to_string(v) + "ULL"; }

// The constexpr shape of d (everything the body reads through K).
std::string shape_source(const PipeDesc& d) {
  std::ostringstream o;
  auto I = [&](const char* name, long long v) { o << "  k." << name << " = " << v << ";\n"; };
  o << "namespace gpl_jit {\n__host__ __device__ constexpr gpl::PipeDesc make_shape() {\n  gpl::PipeDesc k{};\n";
  I("ncols", d.ncols);
  I("slot_bytes", d.slot_bytes);
  for (int c = 0; c < d.ncols; c++)
    o << "  k.colw[" << c << "] = " << d.colw[c] << "; k.coloff[" << c << "] = " << d.coloff[c] << "; k.lazy[" << c
      << "] = " << d.lazy[c] << ";\n";
  I("stage_rows", d.stage_rows);
  I("depth", d.depth);
  I("nwarps", d.nwarps);
  I("npack", d.npack);
  I("min_blocks", d.min_blocks);
  I("ndrain", d.ndrain);
  I("flush_each_tile", d.flush_each_tile);
  I("nfilt", d.nfilt);
  I("nsprobe", d.nsprobe);
  I("nprobe", d.nprobe);
  I("npush", d.npush);
  for (int f = 0; f < d.nfilt; f++) {
    const Filt& F = d.filt[f];
    o << "  k.filt[" << f << "] = gpl::Filt{" << F.kind << ", " << F.ref << ", " << i64(F.lo) << ", " << i64(F.hi) << ", "
      << u64(F.mask) << "};\n";
  }
  for (int p = 0; p < d.nprobe; p++) {
    const Probe& P = d.probe[p];
    o << "  k.probe[" << p << "] = gpl::Probe{" << P.ht << ", " << P.kind << ", " << P.k1 << ", " << P.k2 << ", " << P.out << "};\n";
  }
  for (int e = 0; e < d.nfield; e++) {
    o << "  k.push[" << e << "] = gpl::Push{" << d.push[e].kind << ", " << d.push[e].src << "};";
    o << " k.qoff[" << e << "] = " << d.qoff[e] << "; k.qw[" << e << "] = " << d.qw[e] << ";\n";
  }
  I("qbytes", d.qbytes);
  I("rowid_field", d.rowid_field);
  I("cl_probe", d.cl_probe);
  I("cl_col", d.cl_col);
  I("cl_off", d.cl_off);
  I("cl_cap", d.cl_cap);
  I("fan_probe", d.fan_probe);
  for (int f = 0; f < MAXQ; f++)
    o << "  k.qlazy[" << f << "] = " << d.qlazy[f] << "; k.qlazy_at[" << f << "] = " << d.qlazy_at[f] << ";\n";
  I("reg_fields", d.reg_fields);
  I("agg_lanes", d.agg_lanes);
  auto term = [&](const char* arr, int t, const Term& T) {
    o << "  k." << arr << "[" << t << "].sign = " << T.sign << "; k." << arr << "[" << t << "].nfact = " << T.nfact << ";\n";
    for (int f = 0; f < T.nfact; f++)
      o << "  k." << arr << "[" << t << "].f[" << f << "] = gpl::Factor{" << T.f[f].field << ", " << T.f[f].b << ", "
        << i64(T.f[f].a) << "};\n";
  };
  for (int t = 0; t < MAXTERM; t++) o << "  k.term_field[" << t << "] = " << d.term_field[t] << ";\n";
  for (int t = 0; t < d.nterm; t++) {
    term("sterm", t, d.sterm[t]);
    term("term", t, d.term[t]);
  }
  I("nfield", d.nfield);
  I("nresid", d.nresid);
  I("ngroup", d.ngroup);
  I("ngroups_total", d.ngroups_total);
  for (int r = 0; r < d.nresid; r++) {
    const Resid& R = d.resid[r];
    o << "  k.resid[" << r << "].kind = " << R.kind << "; k.resid[" << r << "].a = " << R.a << "; k.resid[" << r
      << "].b = " << R.b << "; k.resid[" << r << "].npairs = " << R.npairs << ";\n";
    for (int i = 0; i < 4; i++)
      o << "  k.resid[" << r << "].pa[" << i << "] = " << R.pa[i] << "; k.resid[" << r << "].pb[" << i << "] = " << R.pb[i] << ";\n";
    o << "  k.resid[" << r << "].lo = " << i64(R.lo) << "; k.resid[" << r << "].hi = " << i64(R.hi) << "; k.resid[" << r
      << "].mask = " << u64(R.mask) << ";\n";
  }
  for (int g = 0; g < d.ngroup; g++) {
    const GroupDim& G = d.gdim[g];
    o << "  k.gdim[" << g << "] = gpl::GroupDim{" << G.field << ", " << G.transform << ", " << G.lo << ", " << G.size << ", "
      << G.stride << ", 0};\n";
  }
  I("nterm", d.nterm);
  I("nagg", d.nagg);
  I("agg_mode", d.agg_mode);
  I("nht", d.nht);
  for (int a = 0; a < d.nagg; a++)
    o << "  k.agg[" << a << "] = gpl::Agg{" << d.agg[a].kind << ", " << d.agg[a].field << ", " << i64(d.agg[a].c) << "};\n";
  for (int h = 0; h < d.nht; h++)
    o << "  k.ht[" << h << "].kind = " << d.ht[h].kind << "; k.ht[" << h << "].hash = " << d.ht[h].hash << "; k.ht[" << h
      << "].width = " << d.ht[h].width << "; k.ht_smem_off[" << h << "] = " << d.ht_smem_off[h] << "; k.ht_smem_bytes["
      << h << "] = " << d.ht_smem_bytes[h] << ";\n";
  for (int h = d.nht; h < MAXHT; h++) o << "  k.ht_smem_off[" << h << "] = -1;\n";
  I("sink", d.sink);
  I("ins_kfield", d.ins_kfield);
  I("ins_pfield", d.ins_pfield);
  I("ins_ptransform", d.ins_ptransform);
  I("ins_width", d.ins_width);
  I("ins_kcol", d.ins_kcol);
  I("ins_dense", d.ins_dense);
  I("ins_q", d.ins_q);
  I("static_tiles", d.static_tiles);
  I("nparts", d.nparts);
  I("part_shift", d.part_shift);
  I("ins_pcol", d.ins_pcol);
  I("ins_psreg", d.ins_psreg);
  I("smem_tables_bytes", d.smem_tables_bytes);
  I("off_queue", d.off_queue);
  I("off_agg", d.off_agg);
  I("off_ring", d.off_ring);
  I("smem_bytes", d.smem_bytes);
  o << "  return k;\n}\n__device__ constexpr gpl::PipeDesc kShape = make_shape();\n}  // namespace gpl_jit\n";
  return o.str();
}

// Launch bounds of the shape: exactly its (warps + 1) x 32 threads and its
// CTAs per SM, so the register budget is the one the configuration can use
// (2 CTAs of 12+1 warps -> <= 78 registers; the generic kernel assumes 1 CTA
// of 17 warps).
std::string program_source(const std::string& shape, int threads, int min_blocks) {
  return "#define GPL_JIT 1\n#include \"common.h\"\n" + shape +
         "#define GPL_SHAPE_OF(d) (::gpl_jit::kShape)\n#include \"pipeline_body.cuh\"\n"
         "extern \"C\" __global__ void __launch_bounds__(" + std::to_string(threads) + ", " +
         std::to_string(min_blocks < 1 ? 1 : min_blocks) + ")\n"
         "gpl_pipeline_jit(const __grid_constant__ gpl::PipeDesc d) { gpl::pipe::pipeline_body(d); }\n";
}

bool compile(const std::string& src, std::vector<char>* cubin, std::string* err) {
  Nvrtc& n = nvrtc();
  if (!n.ok) {
    *err = "NVRTC unavailable: " + n.why;
    return false;
  }
  nvrtcProgram prog = nullptr;
  if (n.create(&prog, src.c_str(), "gpl_pipeline_jit.cu", kJitNumSources, kJitSources, kJitSourceNames) != 0) {
    *err = "nvrtcCreateProgram failed";
    return false;
  }
  const char* opts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", "--extra-device-vectorization"};
  const nvrtcResult rc = n.compile(prog, 4, opts);
  if (rc != 0) {
    size_t ls = 0;
    n.log_size(prog, &ls);
    std::string log(ls, '\0');
    if (ls) n.log(prog, &log[0]);
    *err = "NVRTC compile failed: " + log.substr(0, 2000);
    n.destroy(&prog);
    return false;
  }
  size_t cs = 0;
  n.cubin_size(prog, &cs);
  cubin->resize(cs);
  n.cubin(prog, cubin->data());
  n.destroy(&prog);
  if (const char* dir = std::getenv("GPL_JIT_DUMP")) {  // diagnostics: cuobjdump / nvdisasm the plan kernels
    static int seq = 0;
    const std::string fn = std::string(dir) + "/gpl_jit_" + std::to_string(seq++) + ".cubin";
    if (FILE* f = std::fopen(fn.c_str(), "wb")) {
      std::fwrite(cubin->data(), 1, cubin->size(), f);
      std::fclose(f);
    }
    if (FILE* f = std::fopen((fn + ".cu").c_str(), "wb")) {
      std::fwrite(src.data(), 1, src.size(), f);
      std::fclose(f);
    }
  }
  return cs > 0;
}

}  // namespace

bool jit_available() { return nvrtc().ok; }

bool jit_prepare(const PipeDesc& d, bool load, std::string* err) {
  const std::string key = shape_source(d);
  std::lock_guard<std::mutex> lk(g_mu);
  Entry& e = g_cache[key];
  if (!e.err.empty()) {
    *err = e.err;
    return false;
  }
  if (e.cubin.empty() && !compile(program_source(key, (d.nwarps + 1) * 32, d.min_blocks), &e.cubin, &e.err)) {
    *err = e.err;
    return false;
  }
  if (load && !e.kernel) {
    cudaError_t c = cudaLibraryLoadData(&e.lib, e.cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
    if (c == cudaSuccess) c = cudaLibraryGetKernel(&e.kernel, e.lib, "gpl_pipeline_jit");
    if (c == cudaSuccess)
      c = cudaFuncSetAttribute((const void*)e.kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, d.smem_bytes);
    if (c != cudaSuccess) {
      e.err = std::string("loading the JIT kernel: ") + cudaGetErrorString(c);
      e.kernel = nullptr;
      *err = e.err;
      return false;
    }
  }
  return true;
}

const void* jit_pipeline_kernel(const PipeDesc& d, std::string* err) {
  if (!jit_prepare(d, true, err)) return nullptr;
  std::lock_guard<std::mutex> lk(g_mu);
  return (const void*)g_cache[shape_source(d)].kernel;
}

}  // namespace gpl
