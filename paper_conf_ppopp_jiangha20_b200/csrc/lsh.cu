// LSH candidate generation on the GPU (term siglen·nnz + siglen/bsize·N
// + d_max·E) and exact Jaccard of every candidate (reading R15).
//
//   minhash_bandkeys : warp per non-empty row; lane owns hash functions s = lane + 32t,
//                      sweeps the row's columns (broadcast by shuffle) keeping running minima,
//                      then writes one u64 band key per band (bsize 1 or 2: the exact tuple).
//   per band         : radix sort (key, row) — stable, so bucket members stay ascending;
//                      run-length encode -> bucket sizes; chunk cap (R14) -> pair counts;
//                      emit_pairs: thread per bucket member, O(1) output offset.
//   all bands        : radix sort packed pairs + unique  -> E (union over bands, R13/R14).
//   pair_jaccard     : thread per pair, sorted-list merge (binary-search when lopsided).
//   heap order       : sort by (J desc, pair asc) through an exact 64-bit fixed-point key
//                      floor(2^64·inter/uni) (order-preserving for denominators < 2^32), so
//                      the host clustering consumes the initial heap as a sorted cursor.
#include <cub/cub.cuh>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include "internal.h"

namespace sr {
namespace {

// ---- hash family (O3 reading R13): SplitMix64 stream -> (a_s odd, b_s), Murmur3 fmix32
uint64_t next_splitmix(uint64_t& x) {
  x += 0x9E3779B97F4A7C15ull;
  uint64_t z = x;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__device__ __forceinline__ uint32_t mix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85EBCA6Bu;
  h ^= h >> 13;
  h *= 0xC2B2AE35u;
  h ^= h >> 16;
  return h;
}

constexpr int kMaxSigPerLane = 8;  // siglen <= 256

template <int SPL>
__global__ void __launch_bounds__(256) minhash_bandkeys(const int64_t* __restrict__ rowptr,
                                                        const int32_t* __restrict__ col,
                                                        const int32_t* __restrict__ live, int64_t L,
                                                        const uint32_t* __restrict__ ha,
                                                        const uint32_t* __restrict__ hb, int siglen,
                                                        int bsize, uint64_t* __restrict__ keys) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  uint32_t a[SPL], b[SPL];
#pragma unroll
  for (int t = 0; t < SPL; ++t) {
    const int s = lane + 32 * t;
    a[t] = s < siglen ? ha[s] : 0u;
    b[t] = s < siglen ? hb[s] : 0u;
  }
  for (int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < L; w += warps) {
    const int32_t r = live[w];
    const int64_t e0 = rowptr[r], e1 = rowptr[r + 1];
    uint32_t m[SPL];
#pragma unroll
    for (int t = 0; t < SPL; ++t) m[t] = 0xFFFFFFFFu;
    for (int64_t e = e0; e < e1; e += 32) {
      const int n = (int)(e1 - e < 32 ? e1 - e : 32);
      const uint32_t mine = lane < n ? (uint32_t)col[e + lane] : 0u;
      for (int j = 0; j < n; ++j) {
        const uint32_t c = __shfl_sync(0xffffffffu, mine, j);
#pragma unroll
        for (int t = 0; t < SPL; ++t) m[t] = min(m[t], mix32(a[t] * c + b[t]));
      }
    }
#pragma unroll
    for (int t = 0; t < SPL; ++t) {
      const int s = lane + 32 * t;
      if (bsize == 1) {
        if (s < siglen) keys[(int64_t)s * L + w] = m[t];
      } else {  // bsize == 2: band s/2 = (sig[s], sig[s+1]) with s even
        const uint32_t nxt = __shfl_down_sync(0xffffffffu, m[t], 1);
        if ((s & 1) == 0 && s + 1 < siglen)
          keys[(int64_t)(s >> 1) * L + w] = ((uint64_t)m[t] << 32) | nxt;
      }
    }
  }
}

__device__ __forceinline__ int64_t chunk_pairs(int64_t s, int64_t C) {
  if (C <= 0 || C >= s) return s * (s - 1) / 2;
  const int64_t f = s / C, r = s % C;
  return f * (C * (C - 1) / 2) + r * (r - 1) / 2;
}

__global__ void run_pair_counts(const int32_t* __restrict__ run_len, int64_t nruns, int64_t C,
                                int64_t* __restrict__ npairs) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < nruns) npairs[i] = chunk_pairs(run_len[i], C);
}

// element x of run r (start s0, size sz) emits pairs (x, y) for y after x in its chunk
__global__ void emit_pairs(const int32_t* __restrict__ run_of, const int64_t* __restrict__ run_start,
                           const int32_t* __restrict__ run_len, const int64_t* __restrict__ run_off,
                           const int32_t* __restrict__ vals_sorted, const int32_t* __restrict__ live,
                           int64_t L, int64_t C, uint64_t* __restrict__ out) {
  const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (x >= L) return;
  const int32_t r = run_of[x];
  const int64_t sz = run_len[r];
  if (sz < 2) return;
  const int64_t s0 = run_start[r];
  const int64_t cap = (C <= 0 || C >= sz) ? sz : C;
  const int64_t lx = x - s0;
  const int64_t chunk = lx / cap;
  const int64_t cs = chunk * cap;
  const int64_t clen = min(cap, sz - cs);
  const int64_t k = lx - cs;
  int64_t o = run_off[r] + chunk * (cap * (cap - 1) / 2) + k * (clen - 1) - k * (k - 1) / 2;
  const uint64_t me = (uint64_t)(uint32_t)live[vals_sorted[x]];
  for (int64_t y = x + 1; y < s0 + cs + clen; ++y) {
    const uint64_t other = (uint64_t)(uint32_t)live[vals_sorted[y]];
    out[o++] = (me << 32) | other;  // live ids ascending within a bucket => me < other
  }
}

__global__ void mark_runs(const int64_t* __restrict__ run_start, const int32_t* __restrict__ run_len,
                          int64_t nruns, int32_t* __restrict__ run_of) {
  const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= nruns) return;
  const int64_t s0 = run_start[r];
  for (int32_t t = 0; t < run_len[r]; ++t) run_of[s0 + t] = (int32_t)r;
}

__global__ void to_int64(const int32_t* __restrict__ a, int64_t n, int64_t* __restrict__ b) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) b[i] = a[i];
}

// exact order-preserving key of J = n/u: floor(2^64·n/u) (n < u), all-ones for J = 1; stored
// complemented so an ascending sort gives J descending
__device__ __forceinline__ uint64_t jaccard_key(uint32_t n, uint32_t u) {
  uint64_t key;
  if (u == 0 || n == 0) {
    key = 0;
  } else if (n >= u) {
    key = ~0ull;
  } else {
    const uint64_t hi = ((uint64_t)n << 32) / u, r1 = ((uint64_t)n << 32) % u;
    const uint64_t lo = (r1 << 32) / u;
    key = (hi << 32) | lo;
  }
  return ~key;
}

constexpr int64_t kLongPair = 2048;  // pairs with more column entries go to the warp kernel

// thread per pair: sorted-list merge (binary search when lopsided); pairs whose two lists hold
// more than kLongPair entries are queued for pair_jaccard_long (one warp each), so a few hub-row
// pairs (R-MAT rows reach 39,705 nnz) no longer serialise whole warps
__global__ void pair_jaccard(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                             const uint64_t* __restrict__ pairs, int64_t E,
                             uint32_t* __restrict__ inter, uint32_t* __restrict__ uni,
                             uint64_t* __restrict__ jkey, int64_t* __restrict__ long_idx, int* __restrict__ n_long) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= E) return;
  const uint64_t pr = pairs[e];
  const int64_t i = (int64_t)(pr >> 32), j = (int64_t)(pr & 0xFFFFFFFFu);
  const int32_t *a = col + rowptr[i], *ae = col + rowptr[i + 1];
  const int32_t *b = col + rowptr[j], *be = col + rowptr[j + 1];
  int64_t na = ae - a, nb = be - b;
  if (na + nb > kLongPair) {
    long_idx[atomicAdd(n_long, 1)] = e;
    return;
  }
  if (na > nb) {
    const int32_t* t = a; a = b; b = t;
    t = ae; ae = be; be = t;
    const int64_t tn = na; na = nb; nb = tn;
  }
  uint32_t n = 0;
  if (nb > 16 * na) {  // lopsided: binary search each element of the short list
    const int32_t* lo = b;
    for (const int32_t* p = a; p < ae; ++p) {
      const int32_t v = *p;
      const int32_t* L = lo; int64_t cnt = be - lo;
      while (cnt > 0) {
        const int64_t h = cnt >> 1;
        if (L[h] < v) { L += h + 1; cnt -= h + 1; } else { cnt = h; }
      }
      lo = L;
      if (lo < be && *lo == v) { ++n; ++lo; }
    }
  } else {
    while (a < ae && b < be) {
      const int32_t x = *a, y = *b;
      n += (x == y);
      a += (x <= y);
      b += (y <= x);
    }
  }
  const uint32_t u = (uint32_t)(na + nb - n);
  inter[e] = n;
  uni[e] = u;
  jkey[e] = jaccard_key(n, u);
}

// one warp per queued long pair: lanes stride over the shorter list and binary-search the longer
__global__ void pair_jaccard_long(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                                  const uint64_t* __restrict__ pairs, const int64_t* __restrict__ long_idx,
                                  const int* __restrict__ n_long, uint32_t* __restrict__ inter,
                                  uint32_t* __restrict__ uni, uint64_t* __restrict__ jkey) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  const int nl = *n_long;
  for (int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < nl; w += nw) {
    const int64_t e = long_idx[w];
    const uint64_t pr = pairs[e];
    const int64_t i = (int64_t)(pr >> 32), j = (int64_t)(pr & 0xFFFFFFFFu);
    const int32_t *a = col + rowptr[i], *b = col + rowptr[j];
    int64_t na = rowptr[i + 1] - rowptr[i], nb = rowptr[j + 1] - rowptr[j];
    if (na > nb) {
      const int32_t* t = a; a = b; b = t;
      const int64_t tn = na; na = nb; nb = tn;
    }
    uint32_t n = 0;
    for (int64_t t = lane; t < na; t += 32) {
      const int32_t v = a[t];
      int64_t lo = 0, cnt = nb;
      while (cnt > 0) {
        const int64_t h = cnt >> 1;
        if (b[lo + h] < v) { lo += h + 1; cnt -= h + 1; } else { cnt = h; }
      }
      n += (lo < nb && b[lo] == v);
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) n += __shfl_xor_sync(0xffffffffu, n, off);
    if (lane == 0) {
      const uint32_t u = (uint32_t)(na + nb - n);
      inter[e] = n;
      uni[e] = u;
      jkey[e] = jaccard_key(n, u);
    }
  }
}

__global__ void iota_u32(uint32_t* a, int64_t n) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) a[i] = (uint32_t)i;
}

__global__ void gather_by(const uint32_t* __restrict__ idx, int64_t n, const uint64_t* __restrict__ p,
                          const uint32_t* __restrict__ ia, const uint32_t* __restrict__ ua,
                          uint64_t* __restrict__ po, uint32_t* __restrict__ io, uint32_t* __restrict__ uo) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t k = idx[i];
  po[i] = p[k];
  io[i] = ia[k];
  uo[i] = ua[k];
}

inline unsigned blocks(int64_t n, int t) { return (unsigned)std::max<int64_t>(1, (n + t - 1) / t); }

}  // namespace

int d2h_staged(void* dst, const void* src, size_t bytes, cudaStream_t s) {
  // a pageable cudaMemcpy runs at a few GB/s through the driver's staging buffer and first-touches
  // the destination on one thread (r02: 0.15 s for C2's 387 MB of candidates); here the PCIe copy
  // of chunk i+1 overlaps the all-thread copy of chunk i out of a pinned ring
  constexpr size_t kChunk = size_t(16) << 20;
  static std::mutex mu;
  static char* ring = nullptr;
  static cudaEvent_t done[2];
  std::lock_guard<std::mutex> lock(mu);
  if (ring == nullptr) {
    SR_CUDA_TRY(cudaMallocHost(reinterpret_cast<void**>(&ring), 2 * kChunk));
    for (auto& e : done) SR_CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  const size_t n = (bytes + kChunk - 1) / kChunk;
  auto issue = [&](size_t i) -> int {
    const size_t off = i * kChunk, len = std::min(kChunk, bytes - off);
    SR_CUDA_TRY(cudaMemcpyAsync(ring + (i & 1) * kChunk, static_cast<const char*>(src) + off, len,
                                cudaMemcpyDeviceToHost, s));
    SR_CUDA_TRY(cudaEventRecord(done[i & 1], s));
    return SR_OK;
  };
  if (n > 0) SR_TRY(issue(0));
  for (size_t i = 0; i < n; ++i) {
    SR_CUDA_TRY(cudaEventSynchronize(done[i & 1]));
    if (i + 1 < n) SR_TRY(issue(i + 1));  // its slot's previous chunk (i-1) was copied out below
    const size_t off = i * kChunk, len = std::min(kChunk, bytes - off);
    const char* from = ring + (i & 1) * kChunk;
    char* to = static_cast<char*>(dst) + off;
    constexpr size_t kPiece = size_t(1) << 20;
    const int64_t np = (int64_t)((len + kPiece - 1) / kPiece);
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < np; ++k) {
      const size_t o = (size_t)k * kPiece;
      std::memcpy(to + o, from + o, std::min(kPiece, len - o));
    }
  }
  return SR_OK;
}

int lsh_candidates(const int64_t* rowptr_h, const int32_t* col_h, int64_t M, int64_t nnz,
                   const sr_reorder_params& p, cudaStream_t s, HostVec<uint64_t>& pairs_by_j,
                   HostVec<uint32_t>& inter_h, HostVec<uint32_t>& uni_h, int64_t* E_out,
                   HostVec<uint64_t>* pairs_by_key) {
  const bool dbg = getenv("SR_DEBUG_LSH") != nullptr;  // per-phase wall times (syncs the stream)
  double tl = 0;
  auto lap = [&](const char* what) {
    if (!dbg) return;
    cudaStreamSynchronize(s);
    const double t = std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
    if (tl > 0) fprintf(stderr, "lsh: %-28s %.4f s\n", what, t - tl);
    tl = t;
  };
  lap("start");
  pairs_by_j.clear();
  inter_h.clear();
  uni_h.clear();
  *E_out = 0;
  std::vector<int32_t> live;
  live.reserve((size_t)M);
  for (int64_t r = 0; r < M; ++r)
    if (rowptr_h[r + 1] > rowptr_h[r]) live.push_back((int32_t)r);
  const int64_t L = (int64_t)live.size();
  if (L < 2) return SR_OK;
  const int siglen = p.siglen, bsize = p.bsize, nb = siglen / bsize;
  std::vector<uint32_t> ha(siglen), hb(siglen);
  uint64_t st = p.seed;
  for (int t = 0; t < siglen; ++t) {
    ha[t] = (uint32_t)(next_splitmix(st) & 0xFFFFFFFFull) | 1u;
    hb[t] = (uint32_t)(next_splitmix(st) & 0xFFFFFFFFull);
  }
  DevBuf<int64_t> d_rowptr(s);
  DevBuf<int32_t> d_col(s), d_live(s);
  DevBuf<uint32_t> d_a(s), d_b(s);
  SR_TRY(d_rowptr.upload(rowptr_h, (size_t)M + 1, s));
  SR_TRY(d_col.upload(col_h, (size_t)nnz, s));
  SR_TRY(d_live.upload(live, s));
  SR_TRY(d_a.upload(ha, s));
  SR_TRY(d_b.upload(hb, s));
  lap("host prep + uploads");
  DevBuf<uint64_t> keys(s);
  SR_TRY(keys.alloc((size_t)nb * L));
  {
    const int threads = 256;
    const unsigned grid = blocks(L, threads / 32);
    const int spl = (siglen + 31) / 32;
#define SR_MH(S) minhash_bandkeys<S><<<grid, threads, 0, s>>>(d_rowptr.p, d_col.p, d_live.p, L, d_a.p, d_b.p, siglen, bsize, keys.p)
    switch (spl) {
      case 1: SR_MH(1); break;
      case 2: SR_MH(2); break;
      case 3: case 4: SR_MH(4); break;
      default: SR_MH(8); break;
    }
#undef SR_MH
    SR_CUDA_TRY(cudaGetLastError());
  }
  lap("minhash");
  // per band: sort, bucket, emit
  DevBuf<uint64_t> kout(s);
  DevBuf<int32_t> vin(s), vout(s), run_len(s), run_of(s), nruns_d(s);
  DevBuf<uint64_t> run_key(s);
  DevBuf<int64_t> run_start(s), run_npairs(s), run_off(s);
  SR_TRY(kout.alloc(L));
  SR_TRY(vin.alloc(L));
  SR_TRY(vout.alloc(L));
  SR_TRY(run_len.alloc(L));
  SR_TRY(run_of.alloc(L));
  SR_TRY(run_key.alloc(L));
  SR_TRY(run_start.alloc(L + 1));
  SR_TRY(run_npairs.alloc(L + 1));
  SR_TRY(run_off.alloc(L + 1));
  SR_TRY(nruns_d.alloc(1));
  {
    std::vector<int32_t> iota((size_t)L);
    for (int64_t t = 0; t < L; ++t) iota[t] = (int32_t)t;
    SR_CUDA_TRY(cudaMemcpyAsync(vin.p, iota.data(), L * sizeof(int32_t), cudaMemcpyHostToDevice, s));
    SR_CUDA_TRY(cudaStreamSynchronize(s));
  }
  DevBuf<uint8_t> temp(s);
  size_t temp_bytes = 0;
  auto ensure_temp = [&](size_t need) -> int {
    if (need > temp_bytes) {
      SR_TRY(temp.alloc(need));
      temp_bytes = need;
    }
    return SR_OK;
  };
  DevBuf<uint64_t> allpairs(s);
  int64_t cap_pairs = 0, n_pairs = 0;
  const int64_t C = p.max_bucket;
  for (int band = 0; band < nb; ++band) {
    size_t need = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, need, keys.p + (int64_t)band * L, kout.p, vin.p, vout.p, (int)L, 0, 64, s);
    SR_TRY(ensure_temp(need));
    need = temp_bytes;
    SR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(temp.p, need, keys.p + (int64_t)band * L, kout.p, vin.p,
                                                vout.p, (int)L, 0, 64, s));
    need = 0;
    cub::DeviceRunLengthEncode::Encode(nullptr, need, kout.p, run_key.p, run_len.p, nruns_d.p, (int)L, s);
    SR_TRY(ensure_temp(need));
    need = temp_bytes;
    SR_CUDA_TRY(cub::DeviceRunLengthEncode::Encode(temp.p, need, kout.p, run_key.p, run_len.p, nruns_d.p,
                                                   (int)L, s));
    int32_t nruns = 0;
    SR_CUDA_TRY(cudaMemcpyAsync(&nruns, nruns_d.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    SR_CUDA_TRY(cudaStreamSynchronize(s));
    if (nruns == L) continue;  // every bucket is a singleton
    // run starts = exclusive sum of lengths (int64)
    to_int64<<<blocks(nruns, 256), 256, 0, s>>>(run_len.p, nruns, run_npairs.p);
    need = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, need, run_npairs.p, run_start.p, (int)nruns + 0, s);
    SR_TRY(ensure_temp(need));
    need = temp_bytes;
    SR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(temp.p, need, run_npairs.p, run_start.p, (int)nruns, s));
    mark_runs<<<blocks(nruns, 256), 256, 0, s>>>(run_start.p, run_len.p, nruns, run_of.p);
    run_pair_counts<<<blocks(nruns, 256), 256, 0, s>>>(run_len.p, nruns, C, run_npairs.p);
    SR_CUDA_TRY(cudaMemsetAsync(run_npairs.p + nruns, 0, sizeof(int64_t), s));
    need = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, need, run_npairs.p, run_off.p, (int)nruns + 1, s);
    SR_TRY(ensure_temp(need));
    need = temp_bytes;
    SR_CUDA_TRY(cub::DeviceScan::ExclusiveSum(temp.p, need, run_npairs.p, run_off.p, (int)nruns + 1, s));
    int64_t band_pairs = 0;
    SR_CUDA_TRY(cudaMemcpyAsync(&band_pairs, run_off.p + nruns, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    SR_CUDA_TRY(cudaStreamSynchronize(s));
    if (band_pairs == 0) continue;
    if (n_pairs + band_pairs > cap_pairs) {
      int64_t ncap = std::max<int64_t>(2 * cap_pairs, n_pairs + band_pairs);
      ncap = std::max<int64_t>(ncap, 1 << 20);
      DevBuf<uint64_t> bigger(s);
      SR_TRY(bigger.alloc(ncap));
      if (n_pairs)
        SR_CUDA_TRY(cudaMemcpyAsync(bigger.p, allpairs.p, n_pairs * sizeof(uint64_t),
                                    cudaMemcpyDeviceToDevice, s));
      SR_CUDA_TRY(cudaStreamSynchronize(s));
      std::swap(bigger.p, allpairs.p);
      std::swap(bigger.n, allpairs.n);
      cap_pairs = ncap;
    }
    // run_off is relative to this band: shift output pointer
    emit_pairs<<<blocks(L, 256), 256, 0, s>>>(run_of.p, run_start.p, run_len.p, run_off.p, vout.p, d_live.p,
                                              L, C, allpairs.p + n_pairs);
    SR_CUDA_TRY(cudaGetLastError());
    n_pairs += band_pairs;
  }
  lap("bands");
  keys.release();
  if (n_pairs == 0) return SR_OK;
  // union over bands: sort + unique
  DevBuf<uint64_t> sorted(s), uniq(s);
  DevBuf<int64_t> nuniq(s);
  SR_TRY(sorted.alloc(n_pairs));
  {
    size_t need = 0;
    cub::DeviceRadixSort::SortKeys(nullptr, need, allpairs.p, sorted.p, n_pairs, 0, 64, s);
    SR_TRY(ensure_temp(need));
    need = temp_bytes;
    SR_CUDA_TRY(cub::DeviceRadixSort::SortKeys(temp.p, need, allpairs.p, sorted.p, n_pairs, 0, 64, s));
  }
  SR_TRY(nuniq.alloc(1));
  {
    size_t need = 0;
    cub::DeviceSelect::Unique(nullptr, need, sorted.p, allpairs.p, nuniq.p, n_pairs, s);
    SR_TRY(ensure_temp(need));
    need = temp_bytes;
    SR_CUDA_TRY(cub::DeviceSelect::Unique(temp.p, need, sorted.p, allpairs.p, nuniq.p, n_pairs, s));
  }
  lap("pair sort + unique");
  int64_t E = 0;
  SR_CUDA_TRY(cudaMemcpyAsync(&E, nuniq.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  SR_CUDA_TRY(cudaStreamSynchronize(s));
  sorted.release();
  if (pairs_by_key && E > (int64_t(1) << 26)) {  // the clustering's membership index above 2^26 pairs (R9)
    pairs_by_key->resize((size_t)E);
    SR_TRY(d2h_staged(pairs_by_key->data(), allpairs.p, E * sizeof(uint64_t), s));
  }
  // exact Jaccard + heap-order sort
  DevBuf<uint32_t> d_inter(s), d_uni(s), idx_in(s), idx_out(s), i2(s), u2(s);
  DevBuf<uint64_t> jkey(s), jkey_out(s), p2(s);
  SR_TRY(d_inter.alloc(E));
  SR_TRY(d_uni.alloc(E));
  SR_TRY(jkey.alloc(E));
  SR_TRY(jkey_out.alloc(E));
  SR_TRY(idx_in.alloc(E));
  SR_TRY(idx_out.alloc(E));
  DevBuf<int64_t> long_idx(s);
  DevBuf<int> n_long(s);
  SR_TRY(long_idx.alloc(E));
  SR_TRY(n_long.alloc(1));
  SR_CUDA_TRY(cudaMemsetAsync(n_long.p, 0, sizeof(int), s));
  pair_jaccard<<<blocks(E, 256), 256, 0, s>>>(d_rowptr.p, d_col.p, allpairs.p, E, d_inter.p, d_uni.p, jkey.p,
                                              long_idx.p, n_long.p);
  pair_jaccard_long<<<1184, 256, 0, s>>>(d_rowptr.p, d_col.p, allpairs.p, long_idx.p, n_long.p, d_inter.p, d_uni.p,
                                         jkey.p);
  iota_u32<<<blocks(E, 256), 256, 0, s>>>(idx_in.p, E);
  SR_CUDA_TRY(cudaGetLastError());
  {
    size_t need = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, need, jkey.p, jkey_out.p, idx_in.p, idx_out.p, E, 0, 64, s);
    SR_TRY(ensure_temp(need));
    need = temp_bytes;
    SR_CUDA_TRY(cub::DeviceRadixSort::SortPairs(temp.p, need, jkey.p, jkey_out.p, idx_in.p, idx_out.p, E, 0,
                                                64, s));
  }
  SR_TRY(p2.alloc(E));
  SR_TRY(i2.alloc(E));
  SR_TRY(u2.alloc(E));
  gather_by<<<blocks(E, 256), 256, 0, s>>>(idx_out.p, E, allpairs.p, d_inter.p, d_uni.p, p2.p, i2.p, u2.p);
  SR_CUDA_TRY(cudaGetLastError());
  lap("jaccard + heap sort");
  pairs_by_j.resize((size_t)E);
  inter_h.resize((size_t)E);
  uni_h.resize((size_t)E);
  SR_TRY(d2h_staged(pairs_by_j.data(), p2.p, E * sizeof(uint64_t), s));
  SR_TRY(d2h_staged(inter_h.data(), i2.p, E * sizeof(uint32_t), s));
  SR_TRY(d2h_staged(uni_h.data(), u2.p, E * sizeof(uint32_t), s));
  lap("D2H");
  *E_out = E;
  return SR_OK;
}

}  // namespace sr
