// guardian_child.cpp — the supervised child process of the guardian (DESIGN R25, SURVEY §8 row f4;
// the FI controller "detects a crash or hang of the GPU program through the
// return status and a timeout", L1996-2007, L2636-2650).
//
// Runs UNGUARDED single-injection FI&FT runs (hauberk_inject_campaign, mode 2: the faulted thread
// dereferences corrupted addresses itself, no watchdog) one at a time and reports each on stdout:
//
//   READY <golden_us>              setup done; golden FT kernel time (CUDA events, microseconds)
//   BEGIN <n>                      injection n is about to run
//   DONE <n> <cls> <alarm> <fail>  its classified outcome (hk_outcome)
//   CRASH <n> <message>            the CUDA context was lost: exit status 3
//
// A hang never prints DONE; the parent kills the process group after its timeout and restarts the
// child after that injection.  The inputs are re-uploaded before every injection, so a stray
// write of an earlier (non-crashing) injection cannot leak into the next one.
//
// usage: hk_guardian_child <problem.blob> <indices.txt> <start_position>
// blob (little endian, written by guardian.py): "HKGRD01\0", int32 bench, exact, nbits, n_arrays,
// uint64 seed, site_mask, hk_ranges, int32 iargs[8], float fargs[4], then n_arrays x
// {uint64 n_floats, float data[n_floats]}.
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <string>
#include <vector>

#include "../../include/hauberk.h"

namespace {

struct Blob {
  int32_t bench = 0, exact = 0, nbits = 1;
  uint64_t seed = 0, site_mask = 0;
  hk_ranges ranges{};
  int32_t iargs[8]{};
  float fargs[4]{};
  std::vector<std::vector<float>> arrays;
};

bool read_exact(FILE* f, void* p, size_t n) { return fread(p, 1, n, f) == n; }

bool load_blob(const char* path, Blob* B) {
  FILE* f = fopen(path, "rb");
  if (!f) return false;
  char magic[8];
  int32_t hdr[4];
  bool ok = read_exact(f, magic, 8) && memcmp(magic, "HKGRD01", 8) == 0 && read_exact(f, hdr, sizeof hdr) &&
            read_exact(f, &B->seed, 8) && read_exact(f, &B->site_mask, 8) && read_exact(f, &B->ranges, sizeof B->ranges) &&
            read_exact(f, B->iargs, sizeof B->iargs) && read_exact(f, B->fargs, sizeof B->fargs);
  if (ok) {
    B->bench = hdr[0]; B->exact = hdr[1]; B->nbits = hdr[2];
    for (int a = 0; ok && a < hdr[3]; ++a) {
      uint64_t n = 0;
      ok = read_exact(f, &n, 8) && n < (1ull << 32);
      if (!ok) break;
      B->arrays.emplace_back((size_t)n);
      ok = read_exact(f, B->arrays.back().data(), (size_t)n * sizeof(float));
    }
  }
  fclose(f);
  return ok;
}

[[noreturn]] void die(int code, const char* what, const char* detail) {
  printf("ERROR %s %s\n", what, detail ? detail : "");
  fflush(stdout);
  exit(code);
}

#define CK(x)                                                    \
  do {                                                           \
    cudaError_t e_ = (x);                                        \
    if (e_ != cudaSuccess) die(2, #x, cudaGetErrorString(e_));   \
  } while (0)

// Device copies of the inputs (re-uploaded per injection) and the outputs / workspaces.
struct Dev {
  std::vector<float*> in;       // one per blob array
  std::vector<size_t> in_bytes;
  float *ws = nullptr, *out0 = nullptr, *out1 = nullptr;
  unsigned long long* hist = nullptr;
  hk_cp_args cp{};
  hk_mriq_args mq{};
  hk_tpacf_args tp{};
  const void* args() const {
    return cp.atoms ? (const void*)&cp : (mq.x ? (const void*)&mq : (const void*)&tp);
  }
};

void setup(const Blob& B, Dev* D) {
  for (const auto& a : B.arrays) {
    float* p = nullptr;
    CK(cudaMalloc(&p, a.size() * sizeof(float) + 16));
    D->in.push_back(p);
    D->in_bytes.push_back(a.size() * sizeof(float));
  }
  const int32_t* I = B.iargs;
  if (B.bench == HK_CP) {
    if (B.arrays.size() != 1) die(2, "blob", "cp needs 1 array");
    const int n = I[0] > 1 ? I[0] : 1;
    CK(cudaMalloc(&D->ws, (size_t)n * 16));
    CK(cudaMalloc(&D->out0, (size_t)I[1] * I[2] * 4));
    D->cp = hk_cp_args{D->in[0], D->ws, I[0], B.fargs[0], B.fargs[1], I[1], I[2], I[3], I[4], I[5], D->out0, B.exact};
  } else if (B.bench == HK_MRIQ) {
    if (B.arrays.size() != 8) die(2, "blob", "mriq needs 8 arrays");
    CK(cudaMalloc(&D->ws, (size_t)(I[1] > 1 ? I[1] : 1) * 16));
    CK(cudaMalloc(&D->out0, (size_t)I[0] * 4));
    CK(cudaMalloc(&D->out1, (size_t)I[0] * 4));
    D->mq = hk_mriq_args{D->in[0], D->in[1], D->in[2], I[0], I[1], D->in[3], D->in[4], D->in[5], D->in[6], D->in[7],
                         D->ws, D->out0, D->out1, B.exact};
  } else if (B.bench == HK_TPACF) {
    if (B.arrays.size() != 2) die(2, "blob", "tpacf needs 2 arrays");
    CK(cudaMalloc(&D->hist, (size_t)(1 + 2 * I[1]) * (I[2] + 2) * 8));
    D->tp = hk_tpacf_args{D->in[0], D->in[1], I[0], I[1], I[2], D->hist};
  } else {
    die(2, "blob", "bad bench");
  }
}

void upload(const Blob& B, const Dev& D, cudaStream_t s) {
  for (size_t a = 0; a < B.arrays.size(); ++a)
    CK(cudaMemcpyAsync(D.in[a], B.arrays[a].data(), D.in_bytes[a], cudaMemcpyHostToDevice, s));
}

double golden_us(const Blob& B, const Dev& D, cudaStream_t s) {
  hk_control* cb = nullptr;
  CK(cudaMalloc(&cb, sizeof(hk_control)));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  float best = 1e30f;
  for (int rep = 0; rep < 3; ++rep) {
    CK(cudaEventRecord(e0, s));
    hk_status st = B.bench == HK_CP     ? hauberk_run_cp(&D.cp, HK_FT, &B.ranges, cb, nullptr, s)
                   : B.bench == HK_MRIQ ? hauberk_run_mriq(&D.mq, HK_FT, &B.ranges, cb, nullptr, s)
                                        : hauberk_run_tpacf(&D.tp, HK_FT, &B.ranges, cb, nullptr, s);
    if (st != HK_OK) die(2, "golden", hauberk_last_error());
    CK(cudaEventRecord(e1, s));
    CK(cudaEventSynchronize(e1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    if (ms < best) best = ms;
  }
  cudaFree(cb);
  return best * 1e3;
}

}  // namespace

int main(int argc, char** argv) {
  if (argc != 4) {
    fprintf(stderr, "usage: %s <problem.blob> <indices.txt> <start_position>\n", argv[0]);
    return 2;
  }
  setvbuf(stdout, nullptr, _IOLBF, 0);
  Blob B;
  if (!load_blob(argv[1], &B)) die(2, "blob", argv[1]);
  std::vector<long long> idx;
  {
    FILE* f = fopen(argv[2], "r");
    if (!f) die(2, "indices", argv[2]);
    long long v;
    while (fscanf(f, "%lld", &v) == 1) idx.push_back(v);
    fclose(f);
  }
  const long start = atol(argv[3]);
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  Dev D;
  setup(B, &D);
  upload(B, D, s);
  printf("READY %.3f\n", golden_us(B, D, s));

  hk_outcome* d_rec = nullptr;
  int64_t* d_counts = nullptr;
  CK(cudaMalloc(&d_rec, sizeof(hk_outcome)));
  CK(cudaMalloc(&d_counts, 15 * sizeof(int64_t)));
  const void* args[3] = {nullptr, nullptr, nullptr};
  const hk_ranges* ranges[3] = {nullptr, nullptr, nullptr};
  args[B.bench] = D.args();
  ranges[B.bench] = &B.ranges;
  for (size_t k = (size_t)(start > 0 ? start : 0); k < idx.size(); ++k) {
    const long long n = idx[k];
    upload(B, D, s);
    CK(cudaMemsetAsync(d_counts, 0, 15 * sizeof(int64_t), s));
    hk_campaign C{};
    C.seed = B.seed; C.first = n; C.count = 1; C.nbits = B.nbits; C.mode = 2; C.batch = 1; C.exact = B.exact;
    C.site_mask[B.bench] = B.site_mask;
    printf("BEGIN %lld\n", n);
    hk_status st = hauberk_inject_campaign(B.bench, args, ranges, &C, d_rec, d_counts, nullptr, s);
    cudaError_t e = st == HK_OK ? cudaStreamSynchronize(s) : cudaSuccess;
    if (st == HK_OK && e == cudaSuccess) e = cudaGetLastError();
    if (st != HK_OK && st != HK_ERR_CUDA && st != HK_ERR_OOM) die(2, "campaign", hauberk_last_error());
    if (st != HK_OK || e != cudaSuccess) {
      const char* why = st != HK_OK ? hauberk_last_error() : cudaGetErrorName(e);
      std::string w = why ? why : "?";
      for (char& c : w) if (c == '\n' || c == ' ') c = '_';
      printf("CRASH %lld %s\n", n, w.c_str());
      fflush(stdout);
      _Exit(3);  // the context is gone: no teardown
    }
    hk_outcome o{};
    CK(cudaMemcpy(&o, d_rec, sizeof o, cudaMemcpyDeviceToHost));
    printf("DONE %lld %d %u %u\n", n, o.cls, o.alarm, o.fail);
  }
  return 0;
}
