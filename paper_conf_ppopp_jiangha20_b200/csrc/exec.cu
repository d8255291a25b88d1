// sm_100a SpMM / SDDMM execution over an ASpT plan (Alg 1, Alg 2
// P:78-92, row-wise GPU mapping P:101, adaptive sparse tiling P:111, Fig 5).
//
// Phase D ("dense tiles"), two engines chosen by the plan's panel height:
//   * panels of > 8 rows: persistent CTAs, a producer warp stages each tile's dense-column rows
//     of B / Y into a shared-memory ring with TMA tile::gather4 (UTMALDG) and bulk copies
//     completing on mbarriers; 8 consumer warps read them per nnz (spmm_dense_kernel,
//     sddmm_dense_kernel);
//   * panels of <= 8 rows: register tiles, one warp per panel keeps every row's accumulator in
//     registers and gathers each dense column's row once (spmm_rtile_kernel, sddmm_rtile_kernel).
// Phase S ("sparse remainder"): row-group tasks in perm2 order, one warp per task,
//   gathers in flight across row boundaries; lanes own 16-byte column fragments, so every
//   gathered row is one coalesced 128-bit load per lane (spmm_task_kernel, sddmm_task_kernel);
//   one-row-per-warp kernels for other K (spmm_sparse_kernel, sddmm_sparse_kernel).
// Lane geometry: LPG lanes cover LPG·VEC columns of one nnz; G = 32/LPG groups of a warp
//   work on G different nnz at once (K = 32 -> 4 nnz per warp instruction).
#include <cuda.h>  // CUtensorMap
#include <cudaTypedefs.h>  // PFN_cuTensorMapEncodeTiled

#include <algorithm>
#include <cstring>
#include <map>
#include <mutex>

#include "internal.h"

namespace sr {
namespace {

constexpr unsigned FULL = 0xffffffffu;

template <int VEC>
struct Frag;
template <>
struct Frag<4> {
  float4 v;
  __device__ __forceinline__ void zero() { v = make_float4(0.f, 0.f, 0.f, 0.f); }
  __device__ __forceinline__ void load_g(const float* p) { v = __ldg(reinterpret_cast<const float4*>(p)); }
  __device__ __forceinline__ void load_cg(const float* p) { v = __ldcg(reinterpret_cast<const float4*>(p)); }
  __device__ __forceinline__ void load_s(const float* p) { v = *reinterpret_cast<const float4*>(p); }
  __device__ __forceinline__ void fma(float a, const Frag& b) {
    v.x = fmaf(a, b.v.x, v.x); v.y = fmaf(a, b.v.y, v.y);
    v.z = fmaf(a, b.v.z, v.z); v.w = fmaf(a, b.v.w, v.w);
  }
  __device__ __forceinline__ void add(const Frag& b) { v.x += b.v.x; v.y += b.v.y; v.z += b.v.z; v.w += b.v.w; }
  __device__ __forceinline__ float dot(const Frag& b) const {
    return fmaf(v.x, b.v.x, fmaf(v.y, b.v.y, fmaf(v.z, b.v.z, v.w * b.v.w)));
  }
  __device__ __forceinline__ void xor_add(int off) {
    v.x += __shfl_xor_sync(FULL, v.x, off); v.y += __shfl_xor_sync(FULL, v.y, off);
    v.z += __shfl_xor_sync(FULL, v.z, off); v.w += __shfl_xor_sync(FULL, v.w, off);
  }
  __device__ __forceinline__ void store(float* p) const { *reinterpret_cast<float4*>(p) = v; }
  __device__ __forceinline__ void store_cs(float* p) const { __stcs(reinterpret_cast<float4*>(p), v); }
};
template <>
struct Frag<1> {
  float v;
  __device__ __forceinline__ void zero() { v = 0.f; }
  __device__ __forceinline__ void load_g(const float* p) { v = __ldg(p); }
  __device__ __forceinline__ void load_cg(const float* p) { v = __ldcg(p); }
  __device__ __forceinline__ void load_s(const float* p) { v = *p; }
  __device__ __forceinline__ void fma(float a, const Frag& b) { v = fmaf(a, b.v, v); }
  __device__ __forceinline__ void add(const Frag& b) { v += b.v; }
  __device__ __forceinline__ float dot(const Frag& b) const { return v * b.v; }
  __device__ __forceinline__ void xor_add(int off) { v += __shfl_xor_sync(FULL, v, off); }
  __device__ __forceinline__ void store(float* p) const { *p = v; }
  __device__ __forceinline__ void store_cs(float* p) const { __stcs(p, v); }
};

// ------------------------------------------------------------------ mbarrier / bulk copy
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// (An L2 evict_last / evict_first split of the gathered rows by access count was measured in
// round 1 and did not help: profiles/r01/NOTES.md.)

// TMA tile::gather4 (sm_100): rows r0..r3 of a 2-D tensor map, box = {columns, 1}, into 4
// consecutive box-sized rows of shared memory (128-byte aligned destination).
__device__ __forceinline__ void tma_gather4(void* dst, const CUtensorMap* map, int col, int r0, int r1, int r2,
                                            int r3, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ char* align128(char* p) {
  return p + ((128 - (smem_u32(p) & 127)) & 127);
}

// ------------------------------------------------------------------ phase S: SpMM
template <int LPG, int VEC, int U, int MINB = 4>
__global__ void __launch_bounds__(256, MINB) spmm_sparse_kernel(
    const Item* __restrict__ items, const uint32_t* __restrict__ meta, int64_t n_items,
    const int2* __restrict__ ent, const float* __restrict__ B, int64_t ldb, float* __restrict__ C,
    int64_t ldc, int K, float* __restrict__ scratch, const int2* __restrict__ split_info,
    int* __restrict__ split_counter) {
  constexpr int G = 32 / LPG;
  constexpr int KC = LPG * VEC;
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  const int64_t it = (int64_t)blockIdx.x * (blockDim.x >> 5) + __shfl_sync(FULL, threadIdx.x >> 5, 0);
  if (it >= n_items) return;
  Item item = items[it];  // warp-uniform through lane-0 shuffles (no divergent-shuffle fallback)
  item.e0 = __shfl_sync(FULL, item.e0, 0); item.e1 = __shfl_sync(FULL, item.e1, 0);
  item.xrow = __shfl_sync(FULL, item.xrow, 0); item.out = __shfl_sync(FULL, item.out, 0);
  const uint32_t mt = __shfl_sync(FULL, meta[it], 0);
  for (int k0 = 0; k0 < K; k0 += KC) {
    const int kk = k0 + lg * VEC;
    const bool kv = kk < K;
    Frag<VEC> acc;
    acc.zero();
    for (int e = item.e0; e < item.e1; e += 32) {
      const int n = min(32, item.e1 - e);
      const int2 my = lane < n ? __ldcs(ent + e + lane) : make_int2(0, 0);
      for (int base = 0; base < n; base += G * U) {
        Frag<VEC> b[U];
        float a[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int j = base + u * G + g;
          const int src = j & 31;
          const int cf = __shfl_sync(FULL, my.x, src);
          const float v = __int_as_float(__shfl_sync(FULL, my.y, src));
          const bool ok = (j < n) && kv;
          a[u] = ok ? v : 0.f;
          if (ok) b[u].load_g(B + (int64_t)cf * ldb + kk); else b[u].zero();
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc.fma(a[u], b[u]);
      }
    }
#pragma unroll
    for (int off = LPG; off < 32; off <<= 1) acc.xor_add(off);
    if (g == 0 && kv) {
      if (mt & kItemSplit) {
        acc.store(scratch + (int64_t)(mt & kItemSlotMask) * K + kk);
      } else {
        float* dst = C + (int64_t)item.out * ldc + kk;
        if (mt & kItemRMW) {
          Frag<VEC> old;
          old.load_cg(dst);
          acc.add(old);
        }
        acc.store_cs(dst);
      }
    }
  }
  if (mt & kItemSplit) {
    // deterministic combine: the last chunk to finish sums all chunk partials in order
    __threadfence();
    __syncwarp();
    const int slot = (int)(mt & kItemSlotMask);
    const int2 si = split_info[slot];
    int last = 0;
    if (lane == 0) last = (atomicAdd(split_counter + si.x, 1) == si.y - 1);
    last = __shfl_sync(FULL, last, 0);
    if (last) {
      __threadfence();
      for (int k = lane * VEC; k < K; k += 32 * VEC) {
        Frag<VEC> s;
        s.zero();
        int c = 0;
        for (; c + 4 <= si.y; c += 4) {  // 4 partial loads in flight, summed in chunk order
          Frag<VEC> p0, p1, p2, p3;
          p0.load_cg(scratch + (int64_t)(si.x + c) * K + k);
          p1.load_cg(scratch + (int64_t)(si.x + c + 1) * K + k);
          p2.load_cg(scratch + (int64_t)(si.x + c + 2) * K + k);
          p3.load_cg(scratch + (int64_t)(si.x + c + 3) * K + k);
          s.add(p0); s.add(p1); s.add(p2); s.add(p3);
        }
        for (; c < si.y; ++c) {
          Frag<VEC> part;
          part.load_cg(scratch + (int64_t)(si.x + c) * K + k);
          s.add(part);
        }
        float* dst = C + (int64_t)item.out * ldc + k;
        if (mt & kItemRMW) {
          Frag<VEC> old;
          old.load_cg(dst);
          s.add(old);
        }
        s.store_cs(dst);
      }
      if (lane == 0) split_counter[si.x] = 0;
    }
  }
}

// ------------------------------------------------------------------ phase S: SDDMM
template <int LPG, int VEC, int U, int NCH, int MINB = 4>
__global__ void __launch_bounds__(256, MINB) sddmm_sparse_kernel(
    const Item* __restrict__ items, int64_t n_items, const int2* __restrict__ ent,
    const int32_t* __restrict__ oidx, const float* __restrict__ X, int64_t ldx,
    const float* __restrict__ Y, int64_t ldy, int K, float* __restrict__ out) {
  constexpr int G = 32 / LPG;
  constexpr int KC = LPG * VEC;
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  const int64_t it = (int64_t)blockIdx.x * (blockDim.x >> 5) + __shfl_sync(FULL, threadIdx.x >> 5, 0);
  if (it >= n_items) return;
  Item item = items[it];  // warp-uniform through lane-0 shuffles (no divergent-shuffle fallback)
  item.e0 = __shfl_sync(FULL, item.e0, 0); item.e1 = __shfl_sync(FULL, item.e1, 0);
  item.xrow = __shfl_sync(FULL, item.xrow, 0);
  Frag<VEC> x[NCH];
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    const int kk = c * KC + lg * VEC;
    if (kk < K) x[c].load_g(X + (int64_t)item.xrow * ldx + kk); else x[c].zero();
  }
  for (int e = item.e0; e < item.e1; e += 32) {
    const int n = min(32, item.e1 - e);
    const int2 my = lane < n ? __ldcs(ent + e + lane) : make_int2(0, 0);
    const int myo = lane < n ? __ldcs(oidx + e + lane) : 0;
    for (int base = 0; base < n; base += G * U) {
      float part[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int j = base + u * G + g;
        const int c = __shfl_sync(FULL, my.x, j & 31);
        const bool ok = j < n;
        float d = 0.f;
#pragma unroll
        for (int ch = 0; ch < NCH; ++ch) {
          const int kk = ch * KC + lg * VEC;
          if (ok && kk < K) {
            Frag<VEC> y;
            y.load_g(Y + (int64_t)c * ldy + kk);
            d += x[ch].dot(y);
          }
        }
        part[u] = d;
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
#pragma unroll
        for (int off = LPG / 2; off > 0; off >>= 1) part[u] += __shfl_xor_sync(FULL, part[u], off);
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int j = base + u * G + g;
        const float v = __int_as_float(__shfl_sync(FULL, my.y, j & 31));
        const int o = __shfl_sync(FULL, myo, j & 31);
        if (lg == 0 && j < n) __stcs(out + o, v * part[u]);
      }
    }
  }
}

// ------------------------------------------------------------------ phase S: SpMM, row-group tasks
// One warp per task = up to 32 consecutive work items (rows in perm2 order, or zero rows) with
// at most task_nnz entries, or one chunk of a split long row (api.cpp: build_tasks).  The warp
// streams the task's entries with U row gathers in flight regardless of where rows end and
// stores each row when its last entry has been added, so the per-row prologue of the one-row-
// per-warp kernel (item descriptor -> entries -> first gather: two dependent latencies) is paid
// once per task and short rows no longer limit the gathers in flight.  Each launch covers 128
// columns (one float4 per lane; the host offsets B and C for K = 128·passes).  Rows are still
// summed in CSR order, chunks of split rows combined in chunk order (deterministic).
template <int U, int VEC>
__device__ __forceinline__ Frag<VEC> task_row_sum(const int2* __restrict__ ent, int e0, int e1, const float* Bk,
                                                  uint32_t ldb) {
  const int lane = threadIdx.x & 31;
  Frag<VEC> acc;
  acc.zero();
  for (int eb = e0; eb < e1; eb += 32) {
    const int n = min(32, e1 - eb);
    const int2 my = lane < n ? __ldcs(ent + eb + lane) : make_int2(0, 0);
    for (int base = 0; base < n; base += U) {
      Frag<VEC> b[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        // past the end: re-load the last entry's row (same lines, no predicate, no zero fill)
        const int c = __shfl_sync(FULL, my.x, min(base + u, n - 1));
        b[u].load_g(reinterpret_cast<const float*>(reinterpret_cast<const char*>(Bk) + (uint64_t)(uint32_t)c * ldb));
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const float a = __int_as_float(__shfl_sync(FULL, my.y, base + u));
        if (base + u < n) acc.fma(a, b[u]);
      }
    }
  }
  return acc;
}

template <int VEC>
__device__ __forceinline__ void task_store(Frag<VEC> v, uint32_t o, float* __restrict__ C, int64_t ldc) {
  float* dst = C + (int64_t)(o & 0x7fffffffu) * ldc + (threadIdx.x & 31) * VEC;
  if (o >> 31) {  // the row also has dense-tile entries (phase D ran first): read-modify-write
    Frag<VEC> old;
    old.load_cg(dst);
    v.add(old);
  }
  v.store_cs(dst);
}

// VEC 4: a launch covers 128 columns (one float4 per lane); VEC 1: 32 columns (K = 32·passes,
// one float per lane, 128-byte gathers).  The host offsets B and C per pass; ldb is in bytes.
template <int U, int VEC>
__device__ __forceinline__ void spmm_task(
    int64_t w, const int4* __restrict__ tasks, const Item* __restrict__ items,
    const uint32_t* __restrict__ meta, const int2* __restrict__ ent, const float* __restrict__ B, uint32_t ldb,
    float* __restrict__ C, int64_t ldc, int K, int k0, float* __restrict__ scratch,
    const int2* __restrict__ split_info, int* __restrict__ split_counter) {
  const int lane = threadIdx.x & 31;
  // warp-uniform values through lane-0 shuffles, so the compiler sees uniform control flow
  // (no divergent-shuffle fallback paths and no stack frame)
  int4 t = __ldg(tasks + w);  // {e0, e1, first item, end item}
  t.x = __shfl_sync(FULL, t.x, 0); t.y = __shfl_sync(FULL, t.y, 0);
  t.z = __shfl_sync(FULL, t.z, 0); t.w = __shfl_sync(FULL, t.w, 0);
  const float* Bk = B + lane * VEC;
  const uint32_t m0 = __ldg(meta + t.z);
  if (m0 & kItemSplit) {  // one chunk of a long row -> scratch; the last chunk combines in order
    const Frag<VEC> acc = task_row_sum<U, VEC>(ent, t.x, t.y, Bk, ldb);
    float* sc = scratch + k0 + lane * VEC;
    acc.store(sc + (int64_t)(m0 & kItemSlotMask) * K);
    __threadfence();
    __syncwarp();
    const int2 si = __ldg(split_info + (m0 & kItemSlotMask));
    int last = 0;
    if (lane == 0) last = (atomicAdd(split_counter + si.x, 1) == si.y - 1);
    last = __shfl_sync(FULL, last, 0);
    if (!last) return;
    __threadfence();
    Frag<VEC> s;
    s.zero();
    int c = 0;
    for (; c + 4 <= si.y; c += 4) {
      Frag<VEC> p[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) p[i].load_cg(sc + (int64_t)(si.x + c + i) * K);
#pragma unroll
      for (int i = 0; i < 4; ++i) s.add(p[i]);
    }
    for (; c < si.y; ++c) {
      Frag<VEC> p;
      p.load_cg(sc + (int64_t)(si.x + c) * K);
      s.add(p);
    }
    const int o = __ldg(reinterpret_cast<const int4*>(items) + t.z).w;
    task_store<VEC>(s, (uint32_t)o | ((m0 & kItemRMW) ? 0x80000000u : 0u), C, ldc);
    if (lane == 0) split_counter[si.x] = 0;
    return;
  }
  const int cnt = t.w - t.z;
  int end = 0;
  uint32_t o = 0;  // output row | RMW flag in bit 31
  if (lane < cnt) {
    const int4 it = __ldg(reinterpret_cast<const int4*>(items) + t.z + lane);
    end = it.y - it.x;
    o = (uint32_t)it.w | ((__ldg(meta + t.z + lane) & kItemRMW) ? 0x80000000u : 0u);
  }
  if (t.x == t.y) {  // zero rows (build_tasks never mixes them with non-empty rows)
    Frag<VEC> z;
    z.zero();
    for (int r = 0; r < cnt; ++r) task_store<VEC>(z, __shfl_sync(FULL, o, r), C, ldc);
    return;
  }
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {  // inclusive scan: end of row r relative to the task's e0
    const int v = __shfl_up_sync(FULL, end, d);
    if (lane >= d) end += v;
  }
  Frag<VEC> acc;
  acc.zero();
  int r = 0;
  int row_end = t.x + __shfl_sync(FULL, end, 0);
  for (int eb = t.x; eb < t.y; eb += 32) {
    const int n = min(32, t.y - eb);
    const int2 my = lane < n ? __ldcs(ent + eb + lane) : make_int2(0, 0);
    for (int base = 0; base < n; base += U) {
      Frag<VEC> b[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        // past the end: re-load the last entry's row (same lines, no predicate, no zero fill)
        const int c = __shfl_sync(FULL, my.x, min(base + u, n - 1));
        b[u].load_g(reinterpret_cast<const float*>(reinterpret_cast<const char*>(Bk) + (uint64_t)(uint32_t)c * ldb));
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const float a = __int_as_float(__shfl_sync(FULL, my.y, base + u));
        if (base + u < n) {
          acc.fma(a, b[u]);
          if (eb + base + u + 1 == row_end) {  // row r is complete (rows here are non-empty)
            task_store<VEC>(acc, __shfl_sync(FULL, o, r), C, ldc);
            acc.zero();
            ++r;
            row_end = t.x + __shfl_sync(FULL, end, r & 31);
          }
        }
      }
    }
  }
}

// Work distribution of the task kernels: each warp draws task indices from a ticket counter in
// task (perm2) order until they run out, so a warp that finishes early takes the next task
// instead of idling until its CTA's slowest warp is done (one task per warp left C2 SDDMM at
// 37 % warps active of a 50 % occupancy limit, profiles/r02).  The next ticket is drawn while
// the current task runs.  Every warp draws exactly one ticket past the last task; the warp
// holding the final ticket (n_tasks + warps - 1) resets the counter for the next launch.
__device__ __forceinline__ int64_t first_ticket(int* ticket) {
  int v = 0;
  if ((threadIdx.x & 31) == 0) v = atomicAdd(ticket, 1);
  return __shfl_sync(FULL, v, 0);
}
__device__ __forceinline__ int draw_ticket(int* ticket) {
  return (threadIdx.x & 31) == 0 ? atomicAdd(ticket, 1) : 0;
}
__device__ __forceinline__ void last_ticket_reset(int* ticket, int64_t w, int64_t n_tasks) {
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  if ((threadIdx.x & 31) == 0 && w == n_tasks + nw - 1) *ticket = 0;
}

// DYN false: one task per warp in launch order (task b·8 + w on warp w of CTA b: consecutive,
// similar rows share an SM and its L1), the measured-faster choice for the SpMM kernels and K = 32.
template <int U, int MINB, int VEC, bool DYN>
__global__ void __launch_bounds__(256, MINB) spmm_task_kernel(
    const int4* __restrict__ tasks, int64_t n_tasks, const Item* __restrict__ items,
    const uint32_t* __restrict__ meta, const int2* __restrict__ ent, const float* __restrict__ B, uint32_t ldb,
    float* __restrict__ C, int64_t ldc, int K, int k0, float* __restrict__ scratch,
    const int2* __restrict__ split_info, int* __restrict__ split_counter, int* __restrict__ ticket) {
  if constexpr (!DYN) {
    const int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + __shfl_sync(FULL, threadIdx.x >> 5, 0);
    if (w < n_tasks)
      spmm_task<U, VEC>(w, tasks, items, meta, ent, B, ldb, C, ldc, K, k0, scratch, split_info, split_counter);
    return;
  }
  int64_t w = first_ticket(ticket);
  while (w < n_tasks) {
    const int nxt = draw_ticket(ticket);
    spmm_task<U, VEC>(w, tasks, items, meta, ent, B, ldb, C, ldc, K, k0, scratch, split_info, split_counter);
    w = __shfl_sync(FULL, nxt, 0);
  }
  last_ticket_reset(ticket, w, n_tasks);
}

// ------------------------------------------------------------------ phase S: SDDMM, row-group tasks
// One warp per task = up to kSddmmTaskRows consecutive remainder rows (or one chunk of a long
// row) with at most task_nnz entries.  At task start the lanes copy the task's X rows into the
// warp's shared-memory slots with cp.async (in parallel with the entry load), so the stream of
// Y gathers never waits on a per-row X load.  Geometry as sddmm_sparse_kernel: 8 lanes × NCH
// float4 per nnz (K = 32·NCH), G = 4 nnz per warp step, U steps of gathers in flight; a group
// whose next entry belongs to another row reloads its X fragment from shared memory.
constexpr int kSddmmTaskRows = 8;

__device__ __forceinline__ void cp_async_cg16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// PERM: lane 8g+k holds batch entry 4k+g, so in step s group g's entry (4s+g) sits in its own
// lane 8g+s, which stores the result from its own registers (no value / index shuffles).
template <int NCH, int U, bool PERM>
__device__ __forceinline__ void sddmm_task(
    int64_t w, float4 (*xs)[NCH * 8], const int4* __restrict__ tasks, const Item* __restrict__ items,
    const int2* __restrict__ ent, const int32_t* __restrict__ oidx, const float* __restrict__ X, int64_t ldx,
    const float* __restrict__ Y, uint32_t ldy_bytes, float* __restrict__ out) {
  constexpr int G = 4, LPG = 8;
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  int4 t = __ldg(tasks + w);  // {e0, e1, first item, end item}; warp-uniform via lane-0 shuffles
  t.x = __shfl_sync(FULL, t.x, 0); t.y = __shfl_sync(FULL, t.y, 0);
  t.z = __shfl_sync(FULL, t.z, 0); t.w = __shfl_sync(FULL, t.w, 0);
  const int cnt = t.w - t.z;
  int end = 0, xrow = 0;
  if (lane < cnt) {
    const int4 it = __ldg(reinterpret_cast<const int4*>(items) + t.z + lane);
    end = it.y - it.x;
    xrow = it.z;
  }
#pragma unroll
  for (int d = 1; d < kSddmmTaskRows; d <<= 1) {  // inclusive scan over the (<= 8) rows
    const int v = __shfl_up_sync(FULL, end, d);
    if (lane >= d) end += v;
  }
  for (int r = 0; r < cnt; ++r) {  // stage the task's X rows (K·4 bytes each) in shared memory
    const int xr = __shfl_sync(FULL, xrow, r);
    if (lane < NCH * 8) cp_async_cg16(&xs[r][lane], X + (int64_t)xr * ldx + lane * 4);
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
  const char* Yl = reinterpret_cast<const char*>(Y + lg * 4);
  float4 x[NCH];
  int cur = -1;
  bool staged = false;
  for (int eb = t.x; eb < t.y; eb += 32) {
    const int n = min(32, t.y - eb);
    const int me = PERM ? 4 * lg + g : lane;  // batch entry this lane loads
    const int2 my = me < n ? __ldcs(ent + eb + me) : make_int2(0, 0);
    const int myo = me < n ? __ldcs(oidx + eb + me) : 0;
    // row (within the task) of the entry this lane loaded
    const int rel = eb + me - t.x;
    int myrow = 0;
    for (int r = 0; r < cnt; ++r) myrow += (__shfl_sync(FULL, end, r) <= rel) ? 1 : 0;
    if (!staged) {
      cp_async_wait_all();
      __syncwarp();
      staged = true;
    }
    for (int base = 0; base < n; base += G * U) {
      float4 y[U][NCH];
      int row[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int jj = min(base + u * G + g, n - 1);
        const int src = PERM ? (((jj & 3) << 3) | (jj >> 2)) : jj;
        const int c = __shfl_sync(FULL, my.x, src);
        row[u] = __shfl_sync(FULL, myrow, src);
        const char* yp = Yl + (uint64_t)(uint32_t)c * ldy_bytes;
#pragma unroll
        for (int ch = 0; ch < NCH; ++ch) y[u][ch] = __ldg(reinterpret_cast<const float4*>(yp + ch * 128));
      }
      float part[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (row[u] != cur) {
          cur = row[u];
#pragma unroll
          for (int ch = 0; ch < NCH; ++ch) x[ch] = xs[cur][ch * 8 + lg];
        }
        float d = 0.f;
#pragma unroll
        for (int ch = 0; ch < NCH; ++ch)
          d += fmaf(x[ch].x, y[u][ch].x, fmaf(x[ch].y, y[u][ch].y, fmaf(x[ch].z, y[u][ch].z, x[ch].w * y[u][ch].w)));
        part[u] = d;
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
#pragma unroll
        for (int off = LPG / 2; off > 0; off >>= 1) part[u] += __shfl_xor_sync(FULL, part[u], off);
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int j = base + u * G + g;
        if (PERM) {
          if (lg == (j >> 2) && j < n) __stcs(out + myo, __int_as_float(my.y) * part[u]);
        } else {
          const float v = __int_as_float(__shfl_sync(FULL, my.y, j & 31));
          const int o = __shfl_sync(FULL, myo, j & 31);
          if (lg == 0 && j < n) __stcs(out + o, v * part[u]);
        }
      }
    }
  }
}

template <int NCH, int U, int MINB, bool PERM, bool DYN>
__global__ void __launch_bounds__(256, MINB) sddmm_task_kernel(
    const int4* __restrict__ tasks, int64_t n_tasks, const Item* __restrict__ items, const int2* __restrict__ ent,
    const int32_t* __restrict__ oidx, const float* __restrict__ X, int64_t ldx, const float* __restrict__ Y,
    uint32_t ldy_bytes, float* __restrict__ out, int* __restrict__ ticket) {
  __shared__ float4 xs[8][kSddmmTaskRows][NCH * 8];
  const int wid = __shfl_sync(FULL, threadIdx.x >> 5, 0);
  if constexpr (!DYN) {
    const int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + wid;
    if (w < n_tasks) sddmm_task<NCH, U, PERM>(w, xs[wid], tasks, items, ent, oidx, X, ldx, Y, ldy_bytes, out);
    return;
  }
  int64_t w = first_ticket(ticket);
  while (w < n_tasks) {
    const int nxt = draw_ticket(ticket);
    sddmm_task<NCH, U, PERM>(w, xs[wid], tasks, items, ent, oidx, X, ldx, Y, ldy_bytes, out);
    w = __shfl_sync(FULL, nxt, 0);
    __syncwarp();  // every lane's reads of the staged X rows precede the next task's staging
  }
  last_ticket_reset(ticket, w, n_tasks);
}

// ------------------------------------------------------------------ phase D: register tiles
// The ASpT dense tiles of panels of <= kRtMaxRows (8) rows (P:111 with a warp-sized panel).  One
// warp owns one panel and keeps the accumulators of all its rows in registers (lane owns VEC
// columns of each row): per dense column it gathers the B row ONCE (the column's header in the
// entry stream) and adds it into every panel row that holds the column (row mask), so a column
// shared by ρ rows costs one gather instead of ρ — the reuse ASpT gets from shared memory, here
// without a staging copy or a shared-memory read per nnz (on B200 an LDS.128 of a staged row
// costs the LSU data pipe as much as the L2 gather it replaces).  U columns are in flight.
// Stream: api.cpp build_rt_stream (headers {col | kRtHeader, mask}, values {row, bits}, columns
// never straddle a 32-entry batch).  Rows with dense nnz are written here; phase S (launched
// after, same stream) read-modify-writes the rows that also have remainder nnz.  Each row's
// dense nnz are added in slot order (count desc, column asc).
template <int U, int VEC, int MINB>
__global__ void __launch_bounds__(256, MINB) spmm_rtile_kernel(
    const int4* __restrict__ units, int64_t n_units, const int2* __restrict__ ent,
    const int32_t* __restrict__ dense_out, const float* __restrict__ B, uint32_t ldb, float* __restrict__ C,
    int64_t ldc, int kw, const int2* __restrict__ split, float* __restrict__ scratch, int* __restrict__ counter,
    int K, int k0) {
  constexpr int P = kRtMaxRows;
  const int lane = threadIdx.x & 31;
  const int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + __shfl_sync(FULL, threadIdx.x >> 5, 0);
  if (w >= n_units) return;
  int4 u = __ldg(units + w);  // {e0, e1, first position, rows}; warp-uniform via lane-0 shuffles
  u.x = __shfl_sync(FULL, u.x, 0); u.y = __shfl_sync(FULL, u.y, 0);
  u.z = __shfl_sync(FULL, u.z, 0); u.w = __shfl_sync(FULL, u.w, 0);
  const bool kv = lane * VEC < kw;  // this lane's columns exist (last pass of a ragged K)
  const char* Bk = reinterpret_cast<const char*>(B + (kv ? lane * VEC : 0));
  Frag<VEC> acc[P];
#pragma unroll
  for (int r = 0; r < P; ++r) acc[r].zero();
  for (int eb = u.x; eb < u.y; eb += 32) {
    const int n = min(32, u.y - eb);
    const int2 my = lane < n ? __ldcs(ent + eb + lane) : make_int2(0, 0);
    unsigned hm = __ballot_sync(FULL, lane < n && my.x < 0);
    while (hm) {
      int hl[U];
      Frag<VEC> b[U];
#pragma unroll
      for (int q = 0; q < U; ++q) {
        hl[q] = hm ? __ffs(hm) - 1 : -1;
        hm &= hm - 1;
        if (hl[q] >= 0) {
          const int c = __shfl_sync(FULL, my.x, hl[q]) & 0x7fffffff;
          b[q].load_g(reinterpret_cast<const float*>(Bk + (uint64_t)(uint32_t)c * ldb));
        }
      }
#pragma unroll
      for (int q = 0; q < U; ++q) {
        if (hl[q] >= 0) {
          const uint32_t mask = (uint32_t)__shfl_sync(FULL, my.y, hl[q]);
          int pos = hl[q] + 1;
#pragma unroll
          for (int r = 0; r < P; ++r) {
            if (mask & (1u << r)) {
              acc[r].fma(__int_as_float(__shfl_sync(FULL, my.y, pos)), b[q]);
              ++pos;
            }
          }
        }
      }
    }
  }
  const int orow = lane < u.w ? __ldg(dense_out + u.z + lane) : -1;
  const int2 sp = __ldg(split + w);
  if (sp.x >= 0) {  // one chunk of a hub panel: partials -> scratch; the last chunk adds them in order
    const int c = sp.y >> 16, nch = sp.y & 0xffff;
    float* sc = scratch + (int64_t)(sp.x + c) * P * K + k0 + lane * VEC;
#pragma unroll
    for (int r = 0; r < P; ++r)
      if (kv) acc[r].store(sc + (int64_t)r * K);
    __threadfence();
    __syncwarp();
    int last = 0;
    if (lane == 0) last = (atomicAdd(counter + sp.x, 1) == nch - 1);
    last = __shfl_sync(FULL, last, 0);
    if (!last) return;
    __threadfence();
#pragma unroll
    for (int r = 0; r < P; ++r) acc[r].zero();
    for (int cc = 0; cc < nch; ++cc) {
      const float* src = scratch + (int64_t)(sp.x + cc) * P * K + k0 + lane * VEC;
#pragma unroll
      for (int r = 0; r < P; ++r) {
        Frag<VEC> part;
        if (kv) part.load_cg(src + (int64_t)r * K); else part.zero();
        acc[r].add(part);
      }
    }
    if (lane == 0) counter[sp.x] = 0;
  }
#pragma unroll
  for (int r = 0; r < P; ++r) {
    const int o = __shfl_sync(FULL, orow, r);
    if (o >= 0 && kv) acc[r].store_cs(C + (int64_t)o * ldc + lane * VEC);
  }
}

// SDDMM over the same register-tile stream: 8-lane groups (K = 32·NCH, lane holds NCH float4 of
// an X row); group g keeps the X fragments of panel rows g and g+4 in registers, so per dense
// column the Y row is gathered once (the four groups read the same addresses: one request) and
// dotted with every panel row of the column's mask that the group owns; 3-step shuffle
// reductions; out[oidx] = a·dot.
template <int NCH, int MINB>
__global__ void __launch_bounds__(256, MINB) sddmm_rtile_kernel(
    const int4* __restrict__ units, int64_t n_units, const int2* __restrict__ ent, const int32_t* __restrict__ oidx,
    const int32_t* __restrict__ pos_xrow, const float* __restrict__ X, int64_t ldx, const float* __restrict__ Y,
    uint32_t ldy, int K, float* __restrict__ out, int accumulate) {
  static_assert(kRtMaxRows == 8, "two panel rows per 8-lane group");
  const int lane = threadIdx.x & 31, g = lane >> 3, lg = lane & 7;
  const int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + __shfl_sync(FULL, threadIdx.x >> 5, 0);
  if (w >= n_units) return;
  int4 u = __ldg(units + w);
  u.x = __shfl_sync(FULL, u.x, 0); u.y = __shfl_sync(FULL, u.y, 0);
  u.z = __shfl_sync(FULL, u.z, 0); u.w = __shfl_sync(FULL, u.w, 0);
  float4 x0[NCH], x1[NCH];
  {
    const int r0 = g, r1 = g + 4;
    const float* p0 = X + (int64_t)(r0 < u.w ? __ldg(pos_xrow + u.z + r0) : 0) * ldx;
    const float* p1 = X + (int64_t)(r1 < u.w ? __ldg(pos_xrow + u.z + r1) : 0) * ldx;
#pragma unroll
    for (int ch = 0; ch < NCH; ++ch) {
      const int kk = ch * 32 + lg * 4;
      x0[ch] = kk < K ? __ldg(reinterpret_cast<const float4*>(p0 + kk)) : make_float4(0.f, 0.f, 0.f, 0.f);
      x1[ch] = kk < K ? __ldg(reinterpret_cast<const float4*>(p1 + kk)) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  }
  const char* Yl = reinterpret_cast<const char*>(Y + lg * 4);
  for (int eb = u.x; eb < u.y; eb += 32) {
    const int n = min(32, u.y - eb);
    const int2 my = lane < n ? __ldcs(ent + eb + lane) : make_int2(0, 0);
    const int myo = lane < n ? __ldcs(oidx + eb + lane) : -1;
    unsigned hm = __ballot_sync(FULL, lane < n && my.x < 0);
    while (hm) {
      const int h = __ffs(hm) - 1;
      hm &= hm - 1;
      const int c = __shfl_sync(FULL, my.x, h) & 0x7fffffff;
      const uint32_t mask = (uint32_t)__shfl_sync(FULL, my.y, h);
      float4 y[NCH];
      const char* yp = Yl + (uint64_t)(uint32_t)c * ldy;
#pragma unroll
      for (int ch = 0; ch < NCH; ++ch)
        y[ch] = (ch * 32 + lg * 4 < K) ? __ldg(reinterpret_cast<const float4*>(yp + ch * 128))
                                       : make_float4(0.f, 0.f, 0.f, 0.f);
      const bool has0 = (mask >> g) & 1u, has1 = (mask >> (g + 4)) & 1u;
      float d0 = 0.f, d1 = 0.f;
#pragma unroll
      for (int ch = 0; ch < NCH; ++ch) {
        d0 += fmaf(x0[ch].x, y[ch].x, fmaf(x0[ch].y, y[ch].y, fmaf(x0[ch].z, y[ch].z, x0[ch].w * y[ch].w)));
        d1 += fmaf(x1[ch].x, y[ch].x, fmaf(x1[ch].y, y[ch].y, fmaf(x1[ch].z, y[ch].z, x1[ch].w * y[ch].w)));
      }
#pragma unroll
      for (int off = 4; off > 0; off >>= 1) {
        d0 += __shfl_xor_sync(FULL, d0, off);
        d1 += __shfl_xor_sync(FULL, d1, off);
      }
      // entry lanes of rows g and g+4 in this column: after the header, rows ascending
      const int p0 = h + 1 + __popc(mask & ((1u << g) - 1u));
      const int p1 = h + 1 + __popc(mask & ((1u << (g + 4)) - 1u));
      const float a0 = __int_as_float(__shfl_sync(FULL, my.y, p0 & 31));
      const int o0 = __shfl_sync(FULL, myo, p0 & 31);
      const float a1 = __int_as_float(__shfl_sync(FULL, my.y, p1 & 31));
      const int o1 = __shfl_sync(FULL, myo, p1 & 31);
      if (lg == 0) {  // K > 128: the host runs 128-column chunks, later ones add to out
        if (has0) __stcs(out + o0, a0 * d0 + (accumulate ? __ldcg(out + o0) : 0.f));
        if (has1) __stcs(out + o1, a1 * d1 + (accumulate ? __ldcg(out + o1) : 0.f));
      }
    }
  }
}

// Scalar fallback of sddmm_rtile_kernel (unaligned operands or K % 4 != 0): one warp per panel
// walks its stream; lanes split K; 5-step reduction.
__global__ void __launch_bounds__(256) sddmm_rtile_scalar_kernel(
    const int2* __restrict__ ent, const int32_t* __restrict__ oidx, const int4* __restrict__ units, int64_t n_units,
    const int32_t* __restrict__ pos_xrow, const float* __restrict__ X, int64_t ldx, const float* __restrict__ Y,
    int64_t ldy, int K, float* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + __shfl_sync(FULL, threadIdx.x >> 5, 0);
  if (w >= n_units) return;
  const int4 u = units[w];
  int col = 0, rem = 0;
  for (int e = u.x; e < u.y; ++e) {
    const int2 v = ent[e];
    if (v.x < 0) {
      col = v.x & 0x7fffffff;
      rem = __popc((unsigned)v.y);
      continue;
    }
    if (rem == 0) continue;  // padding
    --rem;
    const float* xr = X + (int64_t)pos_xrow[u.z + v.x] * ldx;
    const float* yr = Y + (int64_t)col * ldy;
    float d = 0.f;
    for (int k = lane; k < K; k += 32) d = fmaf(xr[k], yr[k], d);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) d += __shfl_xor_sync(FULL, d, off);
    if (lane == 0) out[oidx[e]] = __int_as_float(v.y) * d;
  }
}

// ------------------------------------------------------------------ phase D
// Persistent CTAs (2 per SM) walk the work units (DUnit = up to kMaxUnitTiles virtual tiles
// of one panel, VTile) round-robin.  A dedicated producer warp streams every tile of every
// unit of its CTA through an NST-deep shared-memory ring: the tile's B/Y rows (one
// cp.async.bulk per dense column, 16-byte aligned, K·4 bytes), its panel-row offsets (trp),
// its entry block (and SDDMM output indices) and a 32-byte stage header, all completing on
// one full mbarrier with a transaction count.  Consumer warps (16) release stages through
// an empty mbarrier, so consumers never meet at a CTA barrier and unit boundaries cost no
// pipeline drain: unit n+1's tiles stream in while unit n's results are stored.
// Consumer warp w owns the contiguous panel rows [w·RPW, (w+1)·RPW), RPW the smallest of 2, 4, 8,
// 16 that covers the panel (before r02t every panel ran RPW 8 or 16, so 16- and 32-row panels left
// most consumer warps idle).  16 consumer warps (56 registers) measured faster than 8 (96):
// C4 64-row panels, dense_min 8: 3.92 -> 3.56 ms per SpMM (r02t); 3 CTAs x 2 stages was slower.
// (SR_DENSE_WARPS / SR_SPMM_STAGES / SR_DENSE_CTAS: compile-time measurement knobs, see
// profiles/r02/NOTES.md; the defaults are the measured choice)
#ifndef SR_DENSE_WARPS
#define SR_DENSE_WARPS 16
#endif
#ifndef SR_SPMM_STAGES
#define SR_SPMM_STAGES 3
#endif
#ifndef SR_SDDMM_STAGES
#define SR_SDDMM_STAGES 3
#endif
#ifndef SR_DENSE_CTAS
#define SR_DENSE_CTAS 2
#endif
constexpr int kDenseWarps = SR_DENSE_WARPS;  // consumer warps per phase-D CTA (+1 producer warp)
constexpr int kSpmmStages = SR_SPMM_STAGES;
constexpr int kSddmmStages = SR_SDDMM_STAGES;  // SDDMM stages also carry output indices (3 fit since r02aa)
constexpr int kMaxStages = kSpmmStages > kSddmmStages ? kSpmmStages : kSddmmStages;
constexpr int kDenseCtasPerSM = SR_DENSE_CTAS;
constexpr size_t kUnitBlobBytes = kMaxUnitBlobBytes;  // DUnit + VTiles

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void consumers_sync() {  // named barrier over the consumer warps
  asm volatile("bar.sync 1, %0;" ::"n"(kDenseWarps * 32) : "memory");
}

// Stage header written by the producer (plain st.shared before its arrive; the arrive has
// release semantics and the consumers' wait acquire semantics).
struct __align__(16) StageHdr {
  int32_t q0, nrows, split, flags;
  int32_t k0, kw, uid, pad;
};
constexpr int kFirstOfPass = 1, kLastOfPass = 2, kFirstOfUnit = 4, kLastOfUnit = 8, kLastOfCta = 16;

struct StageLayout {
  int b_floats;   // TW × KCP
  int trp_ints;   // TS
  bool oidx;
  int nst;        // pipeline depth (<= kMaxStages)
  int dbg;        // measurement knobs (SR_DEBUG_DENSE): 1 = skip consumer math, 2 = skip copies
  bool bulk;      // TMA bulk copies (16-byte-aligned rows); else the producer copies with LDG/STS
  // stage = [staged rows (128-byte aligned for the tensor TMA)] [trp] [entries] [oidx] [header]
  __host__ __device__ size_t b_off() const { return 0; }
  __host__ __device__ size_t trp_off() const { return b_off() + (size_t)b_floats * 4; }
  __host__ __device__ size_t ent_off() const { return trp_off() + (size_t)trp_ints * 4; }
  __host__ __device__ size_t oidx_off() const { return ent_off() + (size_t)kMaxTileEntries * 8; }
  __host__ __device__ size_t hdr_off() const { return oidx_off() + (oidx ? (size_t)kMaxTileEntries * 4 : 0); }
  __host__ __device__ size_t bytes() const { return (hdr_off() + sizeof(StageHdr) + 127) / 128 * 128; }
  __host__ size_t smem(int nst_) const { return 128 + (size_t)nst_ * bytes() + 2 * kUnitBlobBytes; }
};

static_assert(kMaxExecTile <= 128, "the producer's lanes stage four tile columns each");
static_assert(kMaxUnitTiles <= 32, "the producer holds one VTile of its unit per lane");

// Producer warp: every tile of every unit of this CTA.
__device__ __forceinline__ void dense_produce(const DUnit* __restrict__ units, int n_units,
                                              const VTile* __restrict__ vtiles,
                                              const int32_t* __restrict__ dense_cols,
                                              const int32_t* __restrict__ trp, const int2* __restrict__ ent,
                                              const int32_t* __restrict__ oidx, const float* __restrict__ src,
                                              int64_t ld, int K, int KCP, const StageLayout& L, char* smem,
                                              uint64_t* full, uint64_t* empty, const int4* __restrict__ blobs,
                                              const int2* __restrict__ blob_meta, uint64_t* blob_bar,
                                              const CUtensorMap* tmap) {
  const int lane = threadIdx.x & 31;
  const size_t SB = L.bytes();
  const int npass = (K + KCP - 1) / KCP;
  // This CTA's units are blockIdx.x + k·gridDim.x (units are sorted by decreasing size, so the
  // round robin balances).  A unit's DUnit and VTiles (<= 32, one per lane) are one contiguous
  // 16-byte-aligned blob, fetched by one bulk copy two units ahead into a 2-slot ring; a tile's
  // dense column ids are loaded from global memory before the producer waits for the tile's
  // stage to drain, so their latency hides behind the consumers.
  char* ring = smem + L.nst * SB;
  const int nmine = ((int)blockIdx.x < n_units) ? (n_units - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x : 0;
  auto fetch_blob = [&](int k, int2 m) {
    if (lane == 0) {
      mbar_expect_tx(&blob_bar[k & 1], (uint32_t)m.y);
      bulk_g2s(ring + (k & 1) * kUnitBlobBytes, reinterpret_cast<const char*>(blobs) + (int64_t)m.x * 16,
               (uint32_t)m.y, &blob_bar[k & 1]);
    }
  };
  for (int k = 0; k < 2 && k < nmine; ++k) fetch_blob(k, blob_meta[blockIdx.x + k * gridDim.x]);
  int2 m_next = (2 < nmine) ? blob_meta[blockIdx.x + 2 * gridDim.x] : make_int2(0, 0);
  int idx = 0;
  for (int k = 0; k < nmine; ++k) {
    const int uid = blockIdx.x + k * gridDim.x;
    mbar_wait(&blob_bar[k & 1], (k >> 1) & 1);
    const char* blob = ring + (k & 1) * kUnitBlobBytes;
    const DUnit u = *reinterpret_cast<const DUnit*>(blob);
    const bool last_unit = k == nmine - 1;
    const VTile mine = lane < u.nvt ? reinterpret_cast<const VTile*>(blob + sizeof(DUnit))[lane] : VTile{0, 0, 0, 0};
    for (int pass = 0; pass < npass; ++pass) {
      const int k0 = pass * KCP, kw = min(KCP, K - k0);
      for (int ti = 0; ti < u.nvt; ++ti, ++idx) {
        const int st = idx % L.nst;
        VTile v;
        v.ent0 = __shfl_sync(FULL, mine.ent0, ti);
        v.nent = __shfl_sync(FULL, mine.nent, ti);
        v.col0 = __shfl_sync(FULL, mine.col0, ti);
        v.ncols = __shfl_sync(FULL, mine.ncols, ti);
        // this lane's four column ids (tile columns 4·lane .. 4·lane+3; a ragged group repeats
        // its first row), in flight while the stage drains
        int cid[4] = {0, 0, 0, 0};
        if (lane * 4 < v.ncols) {
#pragma unroll
          for (int q = 0; q < 4; ++q) cid[q] = __ldg(dense_cols + v.col0 + min(lane * 4 + q, v.ncols - 1));
        }
        if (idx >= L.nst) mbar_wait(&empty[st], ((idx - L.nst) / L.nst) & 1);
        char* base = smem + st * SB;
        if (lane == 0) {
          StageHdr* h = reinterpret_cast<StageHdr*>(base + L.hdr_off());
          int f = 0;
          if (ti == 0) f |= kFirstOfPass;
          if (ti == u.nvt - 1) f |= kLastOfPass;
          if (ti == 0 && pass == 0) f |= kFirstOfUnit;
          if (ti == u.nvt - 1 && pass == npass - 1) f |= kLastOfUnit | (last_unit ? kLastOfCta : 0);
          *h = StageHdr{u.q0, u.nrows, u.split, f, k0, kw, uid, 0};
        }
        const int vt = u.vt0 + ti;
        if (L.dbg & 2) {  // measurement knob: no copies
          if (lane == 0) mbar_arrive(&full[st]);
          continue;
        }
        if (!L.bulk) {  // unaligned operands (scalar path): plain loads and shared stores
          float* bs = reinterpret_cast<float*>(base + L.b_off());
          const int32_t* cols = dense_cols + v.col0;
          for (int i = lane; i < v.ncols * kw; i += 32) {
            const int j = i / kw, k = i - j * kw;
            bs[(size_t)j * KCP + k] = __ldg(src + (int64_t)cols[j] * ld + k0 + k);
          }
          int32_t* ts = reinterpret_cast<int32_t*>(base + L.trp_off());
          for (int i = lane; i < L.trp_ints; i += 32) ts[i] = trp[(int64_t)vt * L.trp_ints + i];
          int2* es = reinterpret_cast<int2*>(base + L.ent_off());
          int32_t* os = reinterpret_cast<int32_t*>(base + L.oidx_off());
          for (int i = lane; i < v.nent; i += 32) {
            es[i] = ent[v.ent0 + i];
            if (L.oidx) os[i] = oidx[v.ent0 + i];
          }
          __syncwarp();
          if (lane == 0) mbar_arrive(&full[st]);
          continue;
        }
        const uint32_t row_bytes = tmap ? (uint32_t)(((v.ncols + 3) & ~3) * KCP * 4) : (uint32_t)(v.ncols * kw * 4);
        const uint32_t bytes = row_bytes + (uint32_t)(L.trp_ints * 4 + v.nent * 8 + (L.oidx ? v.nent * 4 : 0));
        if (lane == 0) mbar_expect_tx(&full[st], bytes);
        __syncwarp();
        if (tmap) {
          // TMA gather4: one instruction stages four dense-column rows (box = KCP columns × 1 row
          // of the row-major operand, 4 row coordinates); tiles have <= 64 columns = 16 lanes
          if (lane * 4 < v.ncols)
            tma_gather4(base + L.b_off() + (size_t)lane * 4 * KCP * 4, tmap, k0, cid[0], cid[1], cid[2], cid[3],
                        &full[st]);
        } else {  // one bulk copy per row: lane l stages rows 4l .. 4l+3
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const int j = lane * 4 + q;
            if (j < v.ncols)
              bulk_g2s(base + L.b_off() + (size_t)j * KCP * 4, src + (int64_t)cid[q] * ld + k0, (uint32_t)(kw * 4),
                       &full[st]);
          }
        }
        if (lane == 0)
          bulk_g2s(base + L.trp_off(), trp + (int64_t)vt * L.trp_ints, (uint32_t)(L.trp_ints * 4), &full[st]);
        if (lane == 1 && v.nent > 0) bulk_g2s(base + L.ent_off(), ent + v.ent0, (uint32_t)(v.nent * 8), &full[st]);
        if (lane == 2 && L.oidx && v.nent > 0)
          bulk_g2s(base + L.oidx_off(), oidx + v.ent0, (uint32_t)(v.nent * 4), &full[st]);
      }
    }
    __syncwarp();  // every lane is done with this blob slot
    if (k + 2 < nmine) {
      fetch_blob(k + 2, m_next);
      m_next = (k + 3 < nmine) ? blob_meta[blockIdx.x + (k + 3) * gridDim.x] : make_int2(0, 0);
    }
  }
  (void)units;
  (void)vtiles;
  (void)dense_cols;
}

__device__ __forceinline__ void dense_init_barriers(uint64_t* full, uint64_t* empty) {
  if (threadIdx.x == 0) {
    for (int s = 0; s < kMaxStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], kDenseWarps * 32);  // every consumer lane releases its own reads
    }
    mbar_init(&full[kMaxStages], 1);  // unit-blob ring (producer only)
    mbar_init(&full[kMaxStages + 1], 1);
    fence_mbar_init();
  }
  __syncthreads();
}

// SpMM dense tiles.
template <int LPG, int VEC, int U, int RPW>
__global__ void __launch_bounds__((kDenseWarps + 1) * 32, kDenseCtasPerSM) spmm_dense_kernel(
    const DUnit* __restrict__ units, int n_units, const VTile* __restrict__ vtiles,
    const int32_t* __restrict__ dense_cols, const int32_t* __restrict__ trp, const int2* __restrict__ ent,
    const int32_t* __restrict__ dense_out, const float* __restrict__ B, int64_t ldb, float* __restrict__ C,
    int64_t ldc, int K, int TW, int TS, int P, float* __restrict__ scratch, const int2* __restrict__ split_info,
    int* __restrict__ split_counter, const int4* __restrict__ blobs, const int2* __restrict__ blob_meta,
    const __grid_constant__ CUtensorMap tmap, int use_tmap, int dbg) {
  constexpr int G = 32 / LPG;
  constexpr int KC = LPG * VEC;
  extern __shared__ __align__(128) char smem_raw[];
  char* const smem = align128(smem_raw);
  __shared__ uint64_t full[kMaxStages + 2], empty[kMaxStages];
  __shared__ int last_ticket;
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  const int warp = threadIdx.x >> 5;
  const StageLayout L{((TW + 3) & ~3) * KC, TS, false, kSpmmStages, dbg >> 1, (dbg & 1) != 0};
  dense_init_barriers(full, empty);
  if (warp == kDenseWarps) {
    dense_produce(units, n_units, vtiles, dense_cols, trp, ent, nullptr, B, ldb, K, KC, L, smem, full, empty,
                  blobs, blob_meta, full + kMaxStages, use_tmap ? &tmap : nullptr);
    return;
  }
  const size_t SB = L.bytes();
  const int r0 = warp * RPW;
  Frag<VEC> acc[RPW];
  int out_row = -1;  // lane i < RPW: output row of panel row r0+i (-1: no dense nnz)
  for (int idx = 0;; ++idx) {
    const int st = idx % L.nst;
    mbar_wait(&full[st], (idx / L.nst) & 1);
    const char* base = smem + st * SB;
    const StageHdr hd = *reinterpret_cast<const StageHdr*>(base + L.hdr_off());
    if (hd.flags & kFirstOfUnit)
      out_row = (lane < RPW && r0 + lane < hd.nrows) ? dense_out[hd.q0 + r0 + lane] : -1;
    if (hd.flags & kFirstOfPass) {
#pragma unroll
      for (int i = 0; i < RPW; ++i) acc[i].zero();
    }
    if (!(L.dbg & 1) && r0 < hd.nrows && lg * VEC < hd.kw) {
      // entries and row bounds come straight from shared memory (broadcast loads): per nnz
      // one LDS.64 of (slot, value), one LDS.128 of the staged row, four FFMA
      const float* tcol = reinterpret_cast<const float*>(base + L.b_off()) + lg * VEC;
      const int32_t* rp = reinterpret_cast<const int32_t*>(base + L.trp_off());
      const int2* es = reinterpret_cast<const int2*>(base + L.ent_off());
#pragma unroll
      for (int i = 0; i < RPW; ++i) {
        const int b0 = rp[r0 + i], b1 = rp[r0 + i + 1];
        int e = b0 + g;
        for (; e + (U - 1) * G < b1; e += U * G) {
          int2 en[U];
#pragma unroll
          for (int uu = 0; uu < U; ++uu) en[uu] = es[e + uu * G];
          Frag<VEC> bv[U];
#pragma unroll
          for (int uu = 0; uu < U; ++uu) bv[uu].load_s(tcol + (size_t)en[uu].x * KC);
#pragma unroll
          for (int uu = 0; uu < U; ++uu) acc[i].fma(__int_as_float(en[uu].y), bv[uu]);
        }
        for (; e < b1; e += G) {
          const int2 en = es[e];
          Frag<VEC> bv;
          bv.load_s(tcol + (size_t)en.x * KC);
          acc[i].fma(__int_as_float(en.y), bv);
        }
      }
    }
    mbar_arrive(&empty[st]);  // release: this lane's reads of the stage happen before the refill
    if (hd.flags & kLastOfPass) {
      const int kk = hd.k0 + lg * VEC;
      const bool kv = kk < K;
#pragma unroll
      for (int i = 0; i < RPW; ++i) {
#pragma unroll
        for (int off = LPG; off < 32; off <<= 1) acc[i].xor_add(off);
        const int orow = __shfl_sync(FULL, out_row, i);
        if (r0 + i < hd.nrows && g == 0 && kv) {
          if (hd.split >= 0)
            acc[i].store(scratch + ((int64_t)hd.split * P + r0 + i) * K + kk);
          else if (orow >= 0)
            acc[i].store_cs(C + (int64_t)orow * ldc + kk);
        }
      }
    }
    if ((hd.flags & kLastOfUnit) && hd.split >= 0) {
      // giant panel split over several units: the last unit to finish sums the chunk
      // partials in unit order (deterministic) and writes the panel's dense rows.  Release /
      // acquire through one thread: the consumers' partial stores happen before thread 0's
      // gpu-scope fence (CTA barrier), its ticket follows the fence; the last unit's thread 0
      // fences after its ticket and the barrier orders every consumer's L2 reads (ld.cg) after
      // (one fence per unit instead of one per consumer thread: each is a CCTL.IVALL of L1)
      consumers_sync();
      const int2 si = split_info[hd.split];
      if (threadIdx.x == 0) {
        __threadfence();
        last_ticket = (atomicAdd(split_counter + si.x, 1) == si.y - 1);
        if (last_ticket) __threadfence();
      }
      consumers_sync();
      if (last_ticket) {
        // all consumer threads share the (row, fragment) sums; chunk partials are added
        // in chunk order with 4 loads in flight (a hub panel can have >100 chunks)
        const int kq = (K + VEC - 1) / VEC;
        for (int item = threadIdx.x; item < hd.nrows * kq; item += kDenseWarps * 32) {
          const int r = item / kq, k = (item - r * kq) * VEC;
          const int orow = dense_out[hd.q0 + r];
          if (orow < 0) continue;
          const float* src = scratch + ((int64_t)si.x * P + r) * K + k;
          const int64_t cstride = (int64_t)P * K;
          Frag<VEC> s;
          s.zero();
          int c = 0;
          for (; c + 4 <= si.y; c += 4) {
            Frag<VEC> p0, p1, p2, p3;
            p0.load_cg(src + (c + 0) * cstride);
            p1.load_cg(src + (c + 1) * cstride);
            p2.load_cg(src + (c + 2) * cstride);
            p3.load_cg(src + (c + 3) * cstride);
            s.add(p0); s.add(p1); s.add(p2); s.add(p3);
          }
          for (; c < si.y; ++c) {
            Frag<VEC> p0;
            p0.load_cg(src + c * cstride);
            s.add(p0);
          }
          s.store_cs(C + (int64_t)orow * ldc + k);
        }
        consumers_sync();
        if (threadIdx.x == 0) split_counter[si.x] = 0;
      }
    }
    if (hd.flags & kLastOfCta) break;
  }
}

// SDDMM dense tiles.  Lane geometry as phase S: LPG lanes × NCH chunks of LPG·VEC columns
// cover one nnz (K=128: 8 lanes × 4 float4, 4 nnz per warp step, 3-step shuffle reduction).
// X fragments of the current row come from global memory (L1-resident across the tiles);
// passes after the first (K > 256) accumulate into out (same lane, same order).
template <int LPG, int VEC, int U, int NCH, int RPW>
__global__ void __launch_bounds__((kDenseWarps + 1) * 32, kDenseCtasPerSM) sddmm_dense_kernel(
    const DUnit* __restrict__ units, int n_units, const VTile* __restrict__ vtiles,
    const int32_t* __restrict__ dense_cols, const int32_t* __restrict__ trp, const int2* __restrict__ ent,
    const int32_t* __restrict__ d_oidx, const int32_t* __restrict__ pos_xrow, const float* __restrict__ X,
    int64_t ldx, const float* __restrict__ Y, int64_t ldy, int K, int TW, int TS, float* __restrict__ out,
    const int4* __restrict__ blobs, const int2* __restrict__ blob_meta, const __grid_constant__ CUtensorMap tmap,
    int use_tmap, int dbg, int nst) {
  constexpr int G = 32 / LPG;
  constexpr int KC = LPG * VEC;   // columns of one chunk
  constexpr int KCP = NCH * KC;   // columns staged per pass (slot stride)
  extern __shared__ __align__(128) char smem_raw[];
  char* const smem = align128(smem_raw);
  __shared__ uint64_t full[kMaxStages + 2], empty[kMaxStages];
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  const int warp = threadIdx.x >> 5;
  const StageLayout L{((TW + 3) & ~3) * KCP, TS, true, nst, dbg >> 1, (dbg & 1) != 0};
  dense_init_barriers(full, empty);
  if (warp == kDenseWarps) {
    dense_produce(units, n_units, vtiles, dense_cols, trp, ent, d_oidx, Y, ldy, K, KCP, L, smem, full, empty,
                  blobs, blob_meta, full + kMaxStages, use_tmap ? &tmap : nullptr);
    return;
  }
  const size_t SB = L.bytes();
  const int r0 = warp * RPW;
  int xrow = 0;  // lane i < RPW: X row of panel row r0+i
  for (int idx = 0;; ++idx) {
    const int st = idx % L.nst;
    mbar_wait(&full[st], (idx / L.nst) & 1);
    const char* base = smem + st * SB;
    const StageHdr hd = *reinterpret_cast<const StageHdr*>(base + L.hdr_off());
    if (hd.flags & kFirstOfUnit) xrow = (lane < RPW && r0 + lane < hd.nrows) ? pos_xrow[hd.q0 + r0 + lane] : 0;
    if (!(L.dbg & 1) && r0 < hd.nrows) {
      const float* tile = reinterpret_cast<const float*>(base + L.b_off());
      const int32_t* rp = reinterpret_cast<const int32_t*>(base + L.trp_off());
      const int2* es = reinterpret_cast<const int2*>(base + L.ent_off());
      const int32_t* os = reinterpret_cast<const int32_t*>(base + L.oidx_off());
      const int k0 = hd.k0, kw = hd.kw;
#pragma unroll 1
      for (int i = 0; i < RPW; ++i) {
        const int b0 = rp[r0 + i], b1 = rp[r0 + i + 1];
        const int xr_i = __shfl_sync(FULL, xrow, i);
        if (b0 >= b1) continue;
        Frag<VEC> x[NCH];
        const float* xr = X + (int64_t)xr_i * ldx + k0;
#pragma unroll
        for (int c = 0; c < NCH; ++c) {
          if (c * KC + lg * VEC < kw) x[c].load_g(xr + c * KC + lg * VEC); else x[c].zero();
        }
        for (int bse = b0; bse < b1; bse += G * U) {
          float part[U];
          int2 en[U];
#pragma unroll
          for (int uu = 0; uu < U; ++uu) {
            const int j = bse + uu * G + g;
            en[uu] = j < b1 ? es[j] : make_int2(0, 0);
          }
          // only groups that hold an entry read a staged row, and steps past the row's last
          // entry are skipped (warp-uniform): a row has ~4-5 entries of a tile on C5 against the
          // G·U = 16 slots of a batch, and every idle slot used to read slot 0 of the stage —
          // 10 shared-memory wavefronts per nnz, the SM's shared-memory pipe 90 % busy (r02af)
#pragma unroll
          for (int uu = 0; uu < U; ++uu) {
            float d = 0.f;
            if (bse + uu * G + g < b1) {
#pragma unroll
              for (int c = 0; c < NCH; ++c) {
                if (c * KC + lg * VEC < kw) {
                  Frag<VEC> y;
                  y.load_s(tile + (size_t)en[uu].x * KCP + c * KC + lg * VEC);
                  d += x[c].dot(y);
                }
              }
            }
            part[uu] = d;
          }
#pragma unroll
          for (int uu = 0; uu < U; ++uu) {
            if (bse + uu * G < b1) {
#pragma unroll
              for (int off = LPG / 2; off > 0; off >>= 1) part[uu] += __shfl_xor_sync(FULL, part[uu], off);
            }
          }
          if (lg == 0) {
#pragma unroll
            for (int uu = 0; uu < U; ++uu) {
              const int j = bse + uu * G + g;
              if (j < b1) {
                const int o = os[j];
                float res = __int_as_float(en[uu].y) * part[uu];
                if (k0 > 0) res += out[o];
                out[o] = res;
              }
            }
          }
        }
      }
    }
    mbar_arrive(&empty[st]);  // release: this lane's reads of the stage happen before the refill
    if (hd.flags & kLastOfCta) break;
  }
}

// ------------------------------------------------------------------ host dispatch
inline int next_pow2(int x) {
  int p = 1;
  while (p < x) p <<= 1;
  return p;
}

constexpr int kSparseWarps = 8;

// Phase-D launch knobs: SR_DEBUG_DENSE (measurement only, see StageLayout::dbg) and the
// persistent grid (kDenseCtasPerSM CTAs per SM, never more CTAs than units).
int dense_dbg() {
  static const int v = [] {
    const char* d = getenv("SR_DEBUG_DENSE");
    return d ? (atoi(d) & 3) : 0;
  }();
  return v;
}

// Tensor map of a row-major fp32 operand [rows × K] (leading dimension ld) for tile::gather4:
// box = `box_cols` columns × 1 row.  The driver's encoder is reached through the runtime's
// entry-point query, so libsr does not link libcuda.  SR_GATHER4=0 falls back to per-row
// cp.async.bulk copies.  Returns false when TMA cannot describe the operand.
bool make_row_gather_map(CUtensorMap* map, const float* base, int64_t rows, int64_t K, int64_t ld, int box_cols) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = [] {
    const char* e = getenv("SR_GATHER4");
    if (e && std::string(e) == "0") return (PFN_cuTensorMapEncodeTiled_v12000) nullptr;
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess) {
      cudaGetLastError();
      return (PFN_cuTensorMapEncodeTiled_v12000) nullptr;
    }
    return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  }();
  // gather4 writes 4 box rows per instruction to a 128-byte-aligned destination: the staged
  // row stride (box_cols floats) must keep 4-row groups 128-byte aligned
  if (!encode || rows < 1 || rows >= (1ll << 31) || box_cols > 256 || (box_cols * 16) % 128 != 0 ||
      ((uintptr_t)base % 16) != 0 || (ld * 4) % 16 != 0)
    return false;
  cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(ld * 4)};
  cuuint32_t box[2] = {(cuuint32_t)box_cols, 1};
  cuuint32_t estr[2] = {1, 1};
  return encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, estr,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Per-handle cache of the tensor map (encoded once per operand base / shape, not per call) and a
// process-wide record of the kernels whose dynamic shared-memory limit has been raised on a
// device, so a steady-state sr_spmm / sr_sddmm call does launch work only.
bool cached_row_gather_map(DevPlan& P, CUtensorMap* map, const float* base, int64_t rows, int64_t K, int64_t ld,
                           int box_cols) {
  static_assert(sizeof(CUtensorMap) <= sizeof(P.tmap_bytes), "tensor map cache too small");
  TmapKey key{base, rows, K, ld, box_cols};
  if (!(P.tmap_valid && P.tmap_key == key)) {
    CUtensorMap m;
    P.tmap_ok = make_row_gather_map(&m, base, rows, K, ld, box_cols);
    std::memcpy(P.tmap_bytes, &m, sizeof(m));
    P.tmap_key = key;
    P.tmap_valid = true;
  }
  std::memcpy(map, P.tmap_bytes, sizeof(CUtensorMap));
  return P.tmap_ok;
}

int raise_smem_limit(const void* kern, size_t smem) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, size_t> done;
  int dev = 0;
  SR_CUDA_TRY(cudaGetDevice(&dev));
  std::lock_guard<std::mutex> lock(mu);
  size_t& cur = done[{kern, dev}];
  if (cur >= smem) return SR_OK;
  SR_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cur = smem;
  return SR_OK;
}

// Phase-S kernel choice (measurement knob SR_PHASE_S; profiles/r01/NOTES.md, profiles/r02/NOTES.md):
// 1 (default) = row-group task kernels where K allows them, 0 = one-row-per-warp kernels (also
// the path for K that is not a multiple of 32).
int env_int(const char* name, int dflt) {
  const char* d = getenv(name);
  return d ? atoi(d) : dflt;
}
bool task_kernels() {
  static const bool v = env_int("SR_PHASE_S", 1) != 0;
  return v;
}

int num_sms() {
  static int n = 0;
  if (n == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

// Grid of a ticket-driven task kernel: the CTAs the device holds at once (occupancy × SMs, cached
// per kernel and device), or fewer when there are fewer tasks.
unsigned resident_grid(const void* kern, int64_t n_tasks) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, int> occ;
  int dev = 0;
  cudaGetDevice(&dev);
  int per_sm = 0;
  {
    std::lock_guard<std::mutex> lock(mu);
    auto it = occ.find({kern, dev});
    if (it == occ.end()) {
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kSparseWarps * 32, 0) != cudaSuccess ||
          per_sm < 1)
        per_sm = 1;
      occ[{kern, dev}] = per_sm;
    } else {
      per_sm = it->second;
    }
  }
  const int64_t need = (n_tasks + kSparseWarps - 1) / kSparseWarps;
  return (unsigned)std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)per_sm * num_sms()));
}

int dense_rows_per_warp(int panel_rows) {
  int r = 2;
  while (r < 16 && r * kDenseWarps < panel_rows) r <<= 1;
  return r;
}

template <int LPG, int VEC>
int run_spmm(sr_csr_s* h, const float* B, int64_t K, int64_t ldb, float* C, int64_t ldc,
             cudaStream_t s, int32_t* launches) {
  DevPlan& P = h->plan;
  constexpr int KC = LPG * VEC;
  constexpr int U = (LPG == 32) ? 8 : 4;  // gathers in flight per lane (phase S)
  constexpr int UD = 4;                   // shared-memory reads in flight per lane (phase D)
  if (P.n_rt > 0) {  // register-tile phase D (panels of <= kRtMaxRows rows)
    const unsigned grid = (unsigned)((P.n_rt + kSparseWarps - 1) / kSparseWarps);
    if (P.profiling) SR_TRY(prof_begin(P, 5, s));
    if (P.n_rt_slots > 0 && P.rt_scratch_k < K) {
      SR_TRY(P.rt_scratch.alloc((size_t)P.n_rt_slots * kRtMaxRows * K));
      P.rt_scratch_k = K;
    }
    auto rk = [&](auto kern, int vec) {
      const int pass = 32 * vec;
      for (int64_t k0 = 0; k0 < K; k0 += pass)
        kern<<<grid, kSparseWarps * 32, 0, s>>>(P.rt_units.p, P.n_rt, P.rt_ent.p, P.dense_out.p, B + k0,
                                                 (uint32_t)(ldb * 4), C + k0, ldc, (int)std::min<int64_t>(pass, K - k0),
                                                 P.rt_split.p, P.rt_scratch.p, P.rt_counter.p, (int)K, (int)k0);
    };
    if constexpr (VEC == 4)
      rk(spmm_rtile_kernel<4, 4, 4>, 4);  // 4 columns in flight, 64 registers (profiles/r02 session f-h)
    else
      rk(spmm_rtile_kernel<8, 1, 8>, 1);
    SR_CUDA_TRY(cudaGetLastError());
    if (P.profiling) SR_TRY(prof_end(P, s));
    ++*launches;
  }
  if (P.n_units > 0) {
    const int TW = P.tile_cols;
    const size_t smem =
        StageLayout{((TW + 3) & ~3) * KC, P.trp_stride, false, kSpmmStages, 0, true}.smem(kSpmmStages);
    CUtensorMap tmap;
    const int use_tmap = (VEC == 4 && cached_row_gather_map(P, &tmap, B, h->A.N, K, ldb, KC)) ? 1 : 0;
    if (P.n_dslots > 0 && P.dscratch_k < K) {
      SR_TRY(P.dscratch.alloc((size_t)P.n_dslots * P.panel_rows * K));
      P.dscratch_k = K;
    }
    const unsigned grid = (unsigned)std::min<int64_t>(P.n_units, (int64_t)kDenseCtasPerSM * num_sms());
    const int flags = (VEC == 4 ? 1 : 0) | (dense_dbg() << 1);
    auto launch = [&](auto kern) -> int {
      SR_TRY(raise_smem_limit(reinterpret_cast<const void*>(kern), smem));
      kern<<<grid, (kDenseWarps + 1) * 32, smem, s>>>(
          P.units.p, (int)P.n_units, P.vtiles.p, P.dense_cols.p, P.trp.p, P.d_ent.p, P.dense_out.p, B, ldb, C, ldc,
          (int)K, TW, P.trp_stride, P.panel_rows, P.dscratch.p, P.dsplit_info.p, P.dsplit_counter.p, P.blobs.p,
          P.blob_meta.p, tmap, use_tmap, flags);
      SR_CUDA_TRY(cudaGetLastError());
      return SR_OK;
    };
    if (P.profiling) SR_TRY(prof_begin(P, 1, s));
    // rows per consumer warp: the smallest of 2, 4, 8, 16 that covers the panel
    const int rpw = dense_rows_per_warp(P.panel_rows);
    if (rpw <= 2) SR_TRY(launch(spmm_dense_kernel<LPG, VEC, UD, 2>));
    else if (rpw <= 4) SR_TRY(launch(spmm_dense_kernel<LPG, VEC, UD, 4>));
    else if (rpw <= 8) SR_TRY(launch(spmm_dense_kernel<LPG, VEC, UD, 8>));
    else SR_TRY(launch(spmm_dense_kernel<LPG, VEC, UD, 16>));
    if (P.profiling) SR_TRY(prof_end(P, s));
    ++*launches;
  }
  if (P.n_items > 0) {
    if (P.n_slots > 0 && P.scratch_k < K) {
      SR_TRY(P.scratch.alloc((size_t)P.n_slots * K));
      P.scratch_k = K;
    }
    const unsigned grid = (unsigned)((P.n_items + kSparseWarps - 1) / kSparseWarps);
    if (P.profiling) SR_TRY(prof_begin(P, 2, s));
    // row-group task kernels: K = 128·passes (float4 lanes) or 32·passes (float lanes)
    const int tvec = (VEC == 4 && K % 128 == 0) ? 4 : (K % 32 == 0 ? 1 : 0);
    if (tvec && ldb * 4 < (1ll << 32) && task_kernels() && P.n_tasks > 0) {
      const int pass = 32 * tvec;
      auto tk = [&](auto kern) {
        const unsigned tgrid = (unsigned)((P.n_tasks + kSparseWarps - 1) / kSparseWarps);
        for (int k0 = 0; k0 < K; k0 += pass)
          kern<<<tgrid, kSparseWarps * 32, 0, s>>>(P.tasks.p, P.n_tasks, P.items.p, P.item_meta.p, P.s_ent.p,
                                                    B + k0, (uint32_t)(ldb * 4), C + k0, ldc, (int)K, k0, P.scratch.p,
                                                    P.split_info.p, P.split_counter.p, P.task_ticket.p);
      };
      if (tvec == 4)
        tk(spmm_task_kernel<4, 8, 4, false>);  // U 4 gathers per lane, 8 CTAs (64 warps) per SM
      else
        tk(spmm_task_kernel<8, 8, 1, false>);
      SR_CUDA_TRY(cudaGetLastError());
      if (P.profiling) SR_TRY(prof_end(P, s));
      ++*launches;
      return SR_OK;
    }
    auto go = [&](auto kern) {
      kern<<<grid, kSparseWarps * 32, 0, s>>>(P.items.p, P.item_meta.p, P.n_items, P.s_ent.p, B, ldb, C, ldc, (int)K,
                                               P.scratch.p, P.split_info.p, P.split_counter.p);
    };
    // one row (or chunk) per warp: U=2 gathers per lane at 8 CTAs (64 warps) per SM (profiles/r01)
    go(spmm_sparse_kernel<LPG, VEC, 2, 8>);
    SR_CUDA_TRY(cudaGetLastError());
    if (P.profiling) SR_TRY(prof_end(P, s));
    ++*launches;
  }
  return SR_OK;
}

template <int LPG, int VEC, int NCH>
int run_sddmm(sr_csr_s* h, const float* X, int64_t ldx, const float* Y, int64_t ldy, int64_t K,
              float* out, cudaStream_t s, int32_t* launches) {
  DevPlan& P = h->plan;
  constexpr int KC = LPG * VEC;
  constexpr int U = (LPG == 32) ? 4 : 2;
  constexpr int NCH_D = (LPG == 32) ? 1 : NCH;  // dense: whole K per pass unless K > 256
  if (P.n_rt > 0) {  // register-tile phase D: 128-column chunks (vector path) or a scalar fallback
    if (P.profiling) SR_TRY(prof_begin(P, 6, s));
    const unsigned grid = (unsigned)((P.n_rt + kSparseWarps - 1) / kSparseWarps);
    if constexpr (VEC == 4) {
      for (int64_t k0 = 0; k0 < K; k0 += 128)
        sddmm_rtile_kernel<4, 4><<<grid, kSparseWarps * 32, 0, s>>>(
            P.rt_units.p, P.n_rt, P.rt_ent.p, P.rt_oidx.p, P.pos_xrow.p, X + k0, ldx, Y + k0, (uint32_t)(ldy * 4),
            (int)std::min<int64_t>(128, K - k0), out, k0 > 0 ? 1 : 0);
    } else {
      sddmm_rtile_scalar_kernel<<<grid, kSparseWarps * 32, 0, s>>>(P.rt_ent.p, P.rt_oidx.p, P.rt_units.p, P.n_rt,
                                                                    P.pos_xrow.p, X, ldx, Y, ldy, (int)K, out);
    }
    SR_CUDA_TRY(cudaGetLastError());
    if (P.profiling) SR_TRY(prof_end(P, s));
    ++*launches;
  }
  if (P.n_units > 0) {
    const int TW = P.tile_cols;
    // ring depth: kSddmmStages (3 since the unit blobs shrank, r02ad: −9-11 % per dense nnz on C5)
    // while two CTAs fit an SM, else 2
    const StageLayout SL{((TW + 3) & ~3) * NCH_D * KC, P.trp_stride, true, kSddmmStages, 0, true};
    int nst = kSddmmStages;
    while (nst > 2 && (size_t)kDenseCtasPerSM * (SL.smem(nst) + 1024) > 233472) --nst;
    const size_t smem = SL.smem(nst);
    CUtensorMap tmap;
    const int use_tmap = (VEC == 4 && cached_row_gather_map(P, &tmap, Y, h->A.N, K, ldy, NCH_D * KC)) ? 1 : 0;
    const unsigned grid = (unsigned)std::min<int64_t>(P.n_units, (int64_t)kDenseCtasPerSM * num_sms());
    const int flags = (VEC == 4 ? 1 : 0) | (dense_dbg() << 1);
    auto launch = [&](auto kern) -> int {
      SR_TRY(raise_smem_limit(reinterpret_cast<const void*>(kern), smem));
      kern<<<grid, (kDenseWarps + 1) * 32, smem, s>>>(
          P.units.p, (int)P.n_units, P.vtiles.p, P.dense_cols.p, P.trp.p, P.d_ent.p, P.d_oidx.p, P.pos_xrow.p, X, ldx,
          Y, ldy, (int)K, TW, P.trp_stride, out, P.blobs.p, P.blob_meta.p, tmap, use_tmap, flags, nst);
      SR_CUDA_TRY(cudaGetLastError());
      return SR_OK;
    };
    // entry slots per group and batch of the SDDMM phase-D consumer (measurement knob; 1 measured
    // best: a row holds ~4-5 entries of a tile, C5 dense 1.47 / 1.41 / 1.29 ms at U 4 / 2 / 1, r02ah)
#ifndef SR_SDDMM_DENSE_U
#define SR_SDDMM_DENSE_U 1
#endif
    constexpr int UD = SR_SDDMM_DENSE_U;
    if (P.profiling) SR_TRY(prof_begin(P, 3, s));
    const int rpw = dense_rows_per_warp(P.panel_rows);
    if (rpw <= 2) SR_TRY(launch(sddmm_dense_kernel<LPG, VEC, UD, NCH_D, 2>));
    else if (rpw <= 4) SR_TRY(launch(sddmm_dense_kernel<LPG, VEC, UD, NCH_D, 4>));
    else if (rpw <= 8) SR_TRY(launch(sddmm_dense_kernel<LPG, VEC, UD, NCH_D, 8>));
    else SR_TRY(launch(sddmm_dense_kernel<LPG, VEC, UD, NCH_D, 16>));
    if (P.profiling) SR_TRY(prof_end(P, s));
    ++*launches;
  }
  if (P.n_sitems > 0) {
    const unsigned grid = (unsigned)((P.n_sitems + kSparseWarps - 1) / kSparseWarps);
    if (P.profiling) SR_TRY(prof_begin(P, 4, s));
    if (LPG == 8 && VEC == 4 && NCH <= 4 && K == 32 * NCH && ldy * 4 < (1ll << 32) && task_kernels() &&
        P.n_stasks > 0) {
      auto tk = [&](auto kern, bool dyn) {
        const unsigned tgrid = dyn ? resident_grid(reinterpret_cast<const void*>(kern), P.n_stasks)
                                   : (unsigned)((P.n_stasks + kSparseWarps - 1) / kSparseWarps);
        kern<<<tgrid, kSparseWarps * 32, 0, s>>>(P.stasks.p, P.n_stasks, P.items.p, P.s_ent.p, P.s_oidx.p, X,
                                                  ldx, Y, (uint32_t)(ldy * 4), out, P.task_ticket.p + 1);
      };
      constexpr int NC = NCH > 4 ? 4 : NCH;  // (NCH <= 4 guarded above; keeps NCH 8 instantiable)
      // K = 128: ticket-driven warps (C2: 0.637 -> 0.547 ms under ncu, warps active 37 -> 49 %);
      // K = 32 measured slower that way (0.283 -> 0.325 ms), K = 64 unmeasured: launch order
      if constexpr (NC == 4) tk(sddmm_task_kernel<NC, 2, 4, true, true>, true);
      else tk(sddmm_task_kernel<NC, 2, 4, true, false>, false);
      SR_CUDA_TRY(cudaGetLastError());
      if (P.profiling) SR_TRY(prof_end(P, s));
      ++*launches;
      return SR_OK;
    }
    auto go = [&](auto kern) {
      kern<<<grid, kSparseWarps * 32, 0, s>>>(P.items.p, P.n_sitems, P.s_ent.p, P.s_oidx.p, X, ldx, Y, ldy, (int)K,
                                               out);
    };
    go(sddmm_sparse_kernel<LPG, VEC, U, NCH, 4>);
    SR_CUDA_TRY(cudaGetLastError());
    if (P.profiling) SR_TRY(prof_end(P, s));
    ++*launches;
  }
  return SR_OK;
}

}  // namespace

int prof_begin(DevPlan& P, int kind, cudaStream_t s) {
  if (P.nrec >= 4) return SR_OK;
  for (int i = 0; i < 8; ++i)
    if (!P.ev[i]) SR_CUDA_TRY(cudaEventCreate(&P.ev[i]));
  P.kinds[P.nrec] = kind;
  SR_CUDA_TRY(cudaEventRecord(P.ev[2 * P.nrec], s));
  return SR_OK;
}

int prof_end(DevPlan& P, cudaStream_t s) {
  if (P.nrec >= 4) return SR_OK;
  SR_CUDA_TRY(cudaEventRecord(P.ev[2 * P.nrec + 1], s));
  ++P.nrec;
  return SR_OK;
}

int launch_spmm(sr_csr_s* h, const float* B, int64_t K, int64_t ldb, float* C, int64_t ldc,
                cudaStream_t s, int32_t* launches) {
  *launches = 0;
  h->plan.nrec = 0;
  const bool vec = (K % 4 == 0) && (ldb % 4 == 0) && (ldc % 4 == 0) &&
                   ((uintptr_t)B % 16 == 0) && ((uintptr_t)C % 16 == 0);
  const int VEC = vec ? 4 : 1;
  const int lpg = std::min(32, next_pow2((int)std::min<int64_t>(32, (K + VEC - 1) / VEC)));
#define SR_S(L, V) return run_spmm<L, V>(h, B, K, ldb, C, ldc, s, launches)
  if (vec) {
    switch (lpg) { case 1: SR_S(1, 4); case 2: SR_S(2, 4); case 4: SR_S(4, 4); case 8: SR_S(8, 4); case 16: SR_S(16, 4); default: SR_S(32, 4); }
  } else {
    switch (lpg) { case 1: SR_S(1, 1); case 2: SR_S(2, 1); case 4: SR_S(4, 1); case 8: SR_S(8, 1); case 16: SR_S(16, 1); default: SR_S(32, 1); }
  }
#undef SR_S
}

int launch_sddmm(sr_csr_s* h, const float* X, int64_t ldx, const float* Y, int64_t ldy, int64_t K,
                 float* out, cudaStream_t s, int32_t* launches) {
  *launches = 0;
  h->plan.nrec = 0;
  const bool vec = (K % 4 == 0) && (ldx % 4 == 0) && (ldy % 4 == 0) &&
                   ((uintptr_t)X % 16 == 0) && ((uintptr_t)Y % 16 == 0);
  const int VEC = vec ? 4 : 1;
  const int lpg = std::min(32, next_pow2((int)std::min<int64_t>(32, (K + VEC - 1) / VEC)));
  const int64_t KC = (int64_t)lpg * VEC;
  const int64_t nch = (K + KC - 1) / KC;
  if (nch > 8) {
    set_error("sr_sddmm: K too large (max 1024 on the vector path, 256 on the scalar path)");
    return SR_EUNSUPPORTED;
  }
#define SR_D(L, V, N) return run_sddmm<L, V, N>(h, X, ldx, Y, ldy, K, out, s, launches)
  if (vec) {
    if (K <= 32) {
      switch (lpg) { case 1: SR_D(1, 4, 1); case 2: SR_D(2, 4, 1); case 4: SR_D(4, 4, 1); default: SR_D(8, 4, 1); }
    }
    if (K <= 256) {  // 8 lanes x NCH float4 per nnz: 4 nnz per warp step, 3-step reductions
      const int64_t n8 = (K + 31) / 32;
      if (n8 <= 2) SR_D(8, 4, 2);
      if (n8 <= 4) SR_D(8, 4, 4);
      SR_D(8, 4, 8);
    }
    switch (nch) { case 3: case 4: SR_D(32, 4, 4); default: SR_D(32, 4, 8); }
  } else {
    if (lpg < 32) {
      switch (lpg) { case 1: SR_D(1, 1, 1); case 2: SR_D(2, 1, 1); case 4: SR_D(4, 1, 1); case 8: SR_D(8, 1, 1); default: SR_D(16, 1, 1); }
    }
    switch (nch) { case 1: SR_D(32, 1, 1); case 2: SR_D(32, 1, 2); case 3: case 4: SR_D(32, 1, 4); default: SR_D(32, 1, 8); }
  }
#undef SR_D
}

}  // namespace sr

// ------------------------------------------------------------------ gather helpers (a11)
namespace sr {
namespace {
__global__ void scatter_rows_kernel(const float* __restrict__ src, int64_t lds, const int32_t* __restrict__ rows,
                                    int64_t n, int64_t K, float* __restrict__ dst, int64_t ldd) {
  const int64_t r = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (r >= n) return;
  const int32_t d = rows[r];
  if (d < 0) return;
  for (int64_t k = threadIdx.x & 31; k < K; k += 32) dst[(int64_t)d * ldd + k] = src[r * lds + k];
}
__global__ void scatter_values_kernel(const float* __restrict__ src, const int64_t* __restrict__ ids, int64_t n,
                                      float* __restrict__ dst) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n && ids[i] >= 0) dst[ids[i]] = src[i];
}

// sr_set_values: ent[e].y := vals[oidx[e]] (oidx = the SDDMM output index of each plan entry,
// i.e. the handle's output order; padding entries carry -1)
__global__ void set_values_kernel(int2* __restrict__ ent, const int32_t* __restrict__ oidx, int64_t n,
                                  const float* __restrict__ vals) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t o = __ldg(oidx + e);
    if (o >= 0) ent[e].y = __float_as_int(__ldg(vals + o));
  }
}
}  // namespace

int launch_set_values(int2* ent, const int32_t* oidx, int64_t n, const float* vals, cudaStream_t s) {
  if (n == 0) return SR_OK;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, (int64_t)num_sms() * 8);
  set_values_kernel<<<grid, 256, 0, s>>>(ent, oidx, n, vals);
  SR_CUDA_TRY(cudaGetLastError());
  return SR_OK;
}

int launch_scatter_rows(const float* src, int64_t lds, const int32_t* rows, int64_t n, int64_t K, float* dst,
                        int64_t ldd, cudaStream_t s) {
  if (n == 0) return SR_OK;
  scatter_rows_kernel<<<(unsigned)((n + 7) / 8), 256, 0, s>>>(src, lds, rows, n, K, dst, ldd);
  SR_CUDA_TRY(cudaGetLastError());
  return SR_OK;
}
int launch_scatter_values(const float* src, const int64_t* ids, int64_t n, float* dst, cudaStream_t s) {
  if (n == 0) return SR_OK;
  scatter_values_kernel<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(src, ids, n, dst);
  SR_CUDA_TRY(cudaGetLastError());
  return SR_OK;
}
}  // namespace sr
