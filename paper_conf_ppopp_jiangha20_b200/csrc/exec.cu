// sm_100a SpMM / SDDMM execution over an ASpT plan (Alg 1, Alg 2
// P:78-92, row-wise GPU mapping P:101, adaptive sparse tiling P:111, Fig 5).
//
// Phase D ("dense tiles"): one CTA per row panel that has dense columns.  The B/Y
//   rows of the panel's dense columns are staged into shared memory tile by tile with
//   bulk asynchronous copies (cp.async.bulk -> UBLKCP, completion on an mbarrier with
//   transaction counts), double-buffered so tile t+1 streams in while tile t is used.
//   Warp w owns panel rows w, w+W, ...; each dense nnz is served from shared memory.
// Phase S ("sparse remainder"): one warp per work item = a remainder row
//   in round-2 order (perm2) or a bounded chunk of a long row; lanes own 16-byte column
//   fragments, so every gathered B/Y row is one coalesced 128-bit load per lane; U gathers
//   are in flight per lane.  SDDMM reduces each dot product with warp shuffles.
// Lane geometry: LPG lanes cover LPG·VEC columns of one nnz; G = 32/LPG groups of a warp
//   work on G different nnz at once (K = 32 -> 4 nnz per warp instruction).
#include <algorithm>

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

// ------------------------------------------------------------------ phase S: SpMM
template <int LPG, int VEC, int U>
__global__ void __launch_bounds__(256, 4) spmm_sparse_kernel(
    const Item* __restrict__ items, const uint32_t* __restrict__ meta, int64_t n_items,
    const int2* __restrict__ ent, const float* __restrict__ B, int64_t ldb, float* __restrict__ C,
    int64_t ldc, int K, float* __restrict__ scratch, const int2* __restrict__ split_info,
    int* __restrict__ split_counter) {
  constexpr int G = 32 / LPG;
  constexpr int KC = LPG * VEC;
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  const int64_t it = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (it >= n_items) return;
  const Item item = items[it];
  const uint32_t mt = meta[it];
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
          const int c = __shfl_sync(FULL, my.x, src);
          const float v = __int_as_float(__shfl_sync(FULL, my.y, src));
          const bool ok = (j < n) && kv;
          a[u] = ok ? v : 0.f;
          if (ok) b[u].load_g(B + (int64_t)c * ldb + kk); else b[u].zero();
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
        for (int c = 0; c < si.y; ++c) {
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
template <int LPG, int VEC, int U, int NCH>
__global__ void __launch_bounds__(256) sddmm_sparse_kernel(
    const Item* __restrict__ items, int64_t n_items, const int2* __restrict__ ent,
    const int32_t* __restrict__ oidx, const float* __restrict__ X, int64_t ldx,
    const float* __restrict__ Y, int64_t ldy, int K, float* __restrict__ out) {
  constexpr int G = 32 / LPG;
  constexpr int KC = LPG * VEC;
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  const int64_t it = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (it >= n_items) return;
  const Item item = items[it];
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

// ------------------------------------------------------------------ phase D
// Work unit = up to kMaxUnitTiles virtual tiles of one panel (DUnit / VTile).  A dedicated
// producer warp streams each tile through a 2- or 3-deep shared-memory ring with
// cp.async.bulk (TMA bulk copies, SASS UBLKCP): the tile's B/Y rows (one 16-byte-aligned
// copy of the staged columns per dense column), its panel-row offsets (trp) and its entry
// block (and the SDDMM output indices), all completing on one full mbarrier with a
// transaction count.  Consumer warps release a stage through an empty mbarrier, so they
// never meet at a CTA barrier, and every load in their inner loop hits shared memory.
// Consumer warp w owns the contiguous panel rows [w·RPW, (w+1)·RPW).
constexpr int kDenseWarps = 8;  // consumer warps per phase-D CTA (+1 producer warp)
constexpr int kMaxStages = 3;  // SpMM runs 3 stages, SDDMM 2 (its stages also carry output indices)
constexpr int kSpmmStages = 3;
constexpr int kSddmmStages = 2;
constexpr size_t kUnitColsBytes = (size_t)kMaxUnitTiles * kMaxExecTile * 4;

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

struct StageLayout {
  int b_floats;   // TW × KCP
  int trp_ints;   // TS
  bool oidx;
  int nst;        // pipeline depth (<= kMaxStages)
  __host__ __device__ size_t trp_off() const { return (size_t)b_floats * 4; }
  __host__ __device__ size_t ent_off() const { return trp_off() + (size_t)trp_ints * 4; }
  __host__ __device__ size_t oidx_off() const { return ent_off() + (size_t)kMaxTileEntries * 8; }
  __host__ __device__ size_t bytes() const { return oidx_off() + (oidx ? (size_t)kMaxTileEntries * 4 : 0); }
};

template <bool kBulk, typename Body, typename PassEnd>
__device__ __forceinline__ void dense_pipeline(const DUnit& u, const VTile* __restrict__ vtiles,
                                               const int32_t* __restrict__ dense_cols,
                                               const int32_t* __restrict__ trp, const int2* __restrict__ ent,
                                               const int32_t* __restrict__ oidx, const float* __restrict__ src,
                                               int64_t ld, int K, int KCP, const StageLayout L, char* smem,
                                               uint64_t* full, uint64_t* empty, Body body, PassEnd pass_end) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int npass = (K + KCP - 1) / KCP;
  const int total = npass * u.nvt;
  const size_t SB = L.bytes();
  if constexpr (kBulk) {
    if (warp == kDenseWarps) {  // producer warp
      // the unit's tile descriptors (lane i holds tile i) and its dense column ids (contiguous
      // range, <= kMaxUnitTiles·kMaxExecTile) are fetched once, so issuing a tile needs no
      // dependent global load
      const VTile mine = lane < u.nvt ? vtiles[u.vt0 + lane] : VTile{0, 0, 0, 0};
      const int col_lo = __shfl_sync(FULL, mine.col0, 0);
      const VTile lastv = vtiles[u.vt0 + u.nvt - 1];
      const int ncol_unit = lastv.col0 + lastv.ncols - col_lo;
      const int NST = L.nst;
      int32_t* ucols = reinterpret_cast<int32_t*>(smem + NST * SB);
      for (int j = lane; j < ncol_unit; j += 32) ucols[j] = dense_cols[col_lo + j];
      __syncwarp();
      for (int idx = 0; idx < total; ++idx) {
        const int st = idx % NST;
        if (idx >= NST) mbar_wait(&empty[st], ((idx - NST) / NST) & 1);
        const int pass = idx / u.nvt, ti = idx % u.nvt, vt = u.vt0 + ti;
        const int k0 = pass * KCP, kw = min(KCP, K - k0);
        VTile v;
        v.ent0 = __shfl_sync(FULL, mine.ent0, ti);
        v.nent = __shfl_sync(FULL, mine.nent, ti);
        v.col0 = __shfl_sync(FULL, mine.col0, ti);
        v.ncols = __shfl_sync(FULL, mine.ncols, ti);
        char* base = smem + st * SB;
        const uint32_t bytes = (uint32_t)(v.ncols * kw * 4 + L.trp_ints * 4 + v.nent * 8 + (L.oidx ? v.nent * 4 : 0));
        if (lane == 0) mbar_expect_tx(&full[st], bytes);
        __syncwarp();
        const int32_t* cols = ucols + (v.col0 - col_lo);
        for (int j = lane; j < v.ncols; j += 32)
          bulk_g2s(base + (size_t)j * KCP * 4, src + (int64_t)cols[j] * ld + k0, (uint32_t)(kw * 4), &full[st]);
        if (lane == 0) bulk_g2s(base + L.trp_off(), trp + (int64_t)vt * L.trp_ints, (uint32_t)(L.trp_ints * 4),
                                &full[st]);
        if (lane == 1 && v.nent > 0) bulk_g2s(base + L.ent_off(), ent + v.ent0, (uint32_t)(v.nent * 8), &full[st]);
        if (lane == 2 && L.oidx && v.nent > 0)
          bulk_g2s(base + L.oidx_off(), oidx + v.ent0, (uint32_t)(v.nent * 4), &full[st]);
      }
      return;
    }
    for (int idx = 0; idx < total; ++idx) {
      const int st = idx % L.nst;
      mbar_wait(&full[st], (idx / L.nst) & 1);
      const int pass = idx / u.nvt;
      const int k0 = pass * KCP;
      const char* base = smem + st * SB;
      body(reinterpret_cast<const float*>(base), reinterpret_cast<const int32_t*>(base + L.trp_off()),
           reinterpret_cast<const int2*>(base + L.ent_off()), reinterpret_cast<const int32_t*>(base + L.oidx_off()),
           k0, min(KCP, K - k0));
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[st]);
      if (idx % u.nvt == u.nvt - 1) pass_end(k0);
    }
  } else {
    for (int idx = 0; idx < total; ++idx) {
      const int pass = idx / u.nvt, vt = u.vt0 + idx % u.nvt;
      const int k0 = pass * KCP, kw = min(KCP, K - k0);
      const VTile v = vtiles[vt];
      float* Bs = reinterpret_cast<float*>(smem);
      int32_t* Ts = reinterpret_cast<int32_t*>(smem + L.trp_off());
      int2* Es = reinterpret_cast<int2*>(smem + L.ent_off());
      int32_t* Os = reinterpret_cast<int32_t*>(smem + L.oidx_off());
      __syncthreads();
      for (int i = threadIdx.x; i < v.ncols * kw; i += blockDim.x) {
        const int j = i / kw, k = i % kw;
        Bs[(size_t)j * KCP + k] = __ldg(src + (int64_t)dense_cols[v.col0 + j] * ld + k0 + k);
      }
      for (int i = threadIdx.x; i < L.trp_ints; i += blockDim.x) Ts[i] = trp[(int64_t)vt * L.trp_ints + i];
      for (int i = threadIdx.x; i < v.nent; i += blockDim.x) {
        Es[i] = ent[v.ent0 + i];
        if (L.oidx) Os[i] = oidx[v.ent0 + i];
      }
      __syncthreads();
      if (warp < kDenseWarps) {
        body(Bs, Ts, Es, Os, k0, kw);
        if (idx % u.nvt == u.nvt - 1) pass_end(k0);
      }
    }
  }
}

__device__ __forceinline__ void dense_init_barriers(uint64_t* full, uint64_t* empty) {
  if (threadIdx.x == 0) {
    for (int s = 0; s < kMaxStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], kDenseWarps);
    }
    fence_mbar_init();
  }
  __syncthreads();
}

// SpMM dense tiles.
template <int LPG, int VEC, int U, int RPW, bool kBulk>
__global__ void __launch_bounds__((kDenseWarps + 1) * 32, 2) spmm_dense_kernel(
    const DUnit* __restrict__ units, const VTile* __restrict__ vtiles, const int32_t* __restrict__ dense_cols,
    const int32_t* __restrict__ trp, const int2* __restrict__ ent, const int32_t* __restrict__ drow_ptr,
    const int32_t* __restrict__ pos_out, const float* __restrict__ B, int64_t ldb, float* __restrict__ C,
    int64_t ldc, int K, int TW, int TS, int P, float* __restrict__ scratch, const int2* __restrict__ split_info,
    int* __restrict__ split_counter) {
  constexpr int G = 32 / LPG;
  constexpr int KC = LPG * VEC;
  extern __shared__ __align__(128) char smem[];
  __shared__ uint64_t full[kMaxStages], empty[kMaxStages];
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  const int warp = threadIdx.x >> 5;
  const DUnit u = units[blockIdx.x];
  dense_init_barriers(full, empty);
  const int r0 = warp * RPW;
  Frag<VEC> acc[RPW];
#pragma unroll
  for (int i = 0; i < RPW; ++i) acc[i].zero();
  auto body = [&](const float* tile, const int32_t* rp, const int2* es, const int32_t*, int k0, int kw) {
    if (r0 >= u.nrows) return;
    const bool kv = lg * VEC < kw;
    const int bnd = lane <= RPW ? rp[r0 + lane] : 0;  // row bounds of this warp's rows
    const int e_lo = __shfl_sync(FULL, bnd, 0), e_hi = __shfl_sync(FULL, bnd, RPW);
    for (int e = e_lo; e < e_hi; e += 32) {
      const int n = min(32, e_hi - e);
      const int2 my = lane < n ? es[e + lane] : make_int2(0, 0);
#pragma unroll
      for (int i = 0; i < RPW; ++i) {
        const int a = max(0, __shfl_sync(FULL, bnd, i) - e), b = min(n, __shfl_sync(FULL, bnd, i + 1) - e);
        for (int base = a; base < b; base += G * U) {
          Frag<VEC> bv[U];
          float av[U];
#pragma unroll
          for (int uu = 0; uu < U; ++uu) {
            const int j = base + uu * G + g;
            const int slot = __shfl_sync(FULL, my.x, j & 31);
            const float v = __int_as_float(__shfl_sync(FULL, my.y, j & 31));
            const bool ok = j < b && kv;
            av[uu] = ok ? v : 0.f;
            if (ok) bv[uu].load_s(tile + (size_t)slot * KC + lg * VEC); else bv[uu].zero();
          }
#pragma unroll
          for (int uu = 0; uu < U; ++uu) acc[i].fma(av[uu], bv[uu]);
        }
      }
    }
  };
  auto pass_end = [&](int k0) {
    const int kk = k0 + lg * VEC;
    const bool kv = kk < K;
#pragma unroll
    for (int i = 0; i < RPW; ++i) {
#pragma unroll
      for (int off = LPG; off < 32; off <<= 1) acc[i].xor_add(off);
      const int r = r0 + i;
      if (r < u.nrows && g == 0 && kv) {
        if (u.split >= 0)
          acc[i].store(scratch + ((int64_t)u.split * P + r) * K + kk);
        else if (drow_ptr[u.q0 + r + 1] > drow_ptr[u.q0 + r])
          acc[i].store_cs(C + (int64_t)pos_out[u.q0 + r] * ldc + kk);
      }
      acc[i].zero();
    }
  };
  const StageLayout L{TW * KC, TS, false, kSpmmStages};
  dense_pipeline<kBulk>(u, vtiles, dense_cols, trp, ent, nullptr, B, ldb, K, KC, L, smem, full, empty, body,
                        pass_end);
  if (u.split >= 0) {
    // giant panel split over several units: the last unit to finish sums the chunk
    // partials in unit order (deterministic) and writes the panel's dense rows
    __shared__ int last;
    __threadfence();
    __syncthreads();
    const int2 si = split_info[u.split];
    if (threadIdx.x == 0) last = (atomicAdd(split_counter + si.x, 1) == si.y - 1);
    __syncthreads();
    if (!last) return;
    __threadfence();
    for (int r = warp; r < u.nrows; r += kDenseWarps + 1) {
      if (drow_ptr[u.q0 + r + 1] == drow_ptr[u.q0 + r]) continue;
      for (int k = lane * VEC; k < K; k += 32 * VEC) {
        Frag<VEC> s;
        s.zero();
        for (int c = 0; c < si.y; ++c) {
          Frag<VEC> part;
          part.load_cg(scratch + ((int64_t)(si.x + c) * P + r) * K + k);
          s.add(part);
        }
        s.store_cs(C + (int64_t)pos_out[u.q0 + r] * ldc + k);
      }
    }
    if (threadIdx.x == 0) split_counter[si.x] = 0;
  }
}

// SDDMM dense tiles.  Lane geometry as phase S: LPG lanes × NCH chunks of LPG·VEC columns
// cover one nnz (K=128: 8 lanes × 4 float4, 4 nnz per warp step, 3-step shuffle reduction).
// X fragments of the current row come from global memory (L1-resident across the tiles);
// passes after the first (K > 256) accumulate into out (same lane, same order).
template <int LPG, int VEC, int U, int NCH, int RPW, bool kBulk>
__global__ void __launch_bounds__((kDenseWarps + 1) * 32, 2) sddmm_dense_kernel(
    const DUnit* __restrict__ units, const VTile* __restrict__ vtiles, const int32_t* __restrict__ dense_cols,
    const int32_t* __restrict__ trp, const int2* __restrict__ ent, const int32_t* __restrict__ d_oidx,
    const int32_t* __restrict__ pos_xrow, const float* __restrict__ X, int64_t ldx, const float* __restrict__ Y,
    int64_t ldy, int K, int TW, int TS, float* __restrict__ out) {
  constexpr int G = 32 / LPG;
  constexpr int KC = LPG * VEC;   // columns of one chunk
  constexpr int KCP = NCH * KC;   // columns staged per pass (slot stride)
  extern __shared__ __align__(128) char smem[];
  __shared__ uint64_t full[kMaxStages], empty[kMaxStages];
  const int lane = threadIdx.x & 31, g = lane / LPG, lg = lane % LPG;
  const int warp = threadIdx.x >> 5;
  const DUnit u = units[blockIdx.x];
  dense_init_barriers(full, empty);
  const int r0 = warp * RPW;
  auto body = [&](const float* tile, const int32_t* rp, const int2* es, const int32_t* os, int k0, int kw) {
    if (r0 >= u.nrows) return;
    const int bnd = lane <= RPW ? rp[r0 + lane] : 0;
    const int e_lo = __shfl_sync(FULL, bnd, 0), e_hi = __shfl_sync(FULL, bnd, RPW);
    for (int e = e_lo; e < e_hi; e += 32) {
      const int n = min(32, e_hi - e);
      const int2 my = lane < n ? es[e + lane] : make_int2(0, 0);
      const int myo = lane < n ? os[e + lane] : 0;
#pragma unroll 1
      for (int i = 0; i < RPW; ++i) {
        const int a = max(0, __shfl_sync(FULL, bnd, i) - e), b = min(n, __shfl_sync(FULL, bnd, i + 1) - e);
        if (a >= b) continue;
        Frag<VEC> x[NCH];
        const float* xr = X + (int64_t)pos_xrow[u.q0 + r0 + i] * ldx + k0;
#pragma unroll
        for (int c = 0; c < NCH; ++c) {
          if (c * KC + lg * VEC < kw) x[c].load_g(xr + c * KC + lg * VEC); else x[c].zero();
        }
        for (int base = a; base < b; base += G * U) {
          float part[U];
#pragma unroll
          for (int uu = 0; uu < U; ++uu) {
            const int j = base + uu * G + g;
            const int slot = __shfl_sync(FULL, my.x, j & 31);
            float d = 0.f;
            if (j < b) {
#pragma unroll
              for (int c = 0; c < NCH; ++c) {
                if (c * KC + lg * VEC < kw) {
                  Frag<VEC> y;
                  y.load_s(tile + (size_t)slot * KCP + c * KC + lg * VEC);
                  d += x[c].dot(y);
                }
              }
            }
            part[uu] = d;
          }
#pragma unroll
          for (int uu = 0; uu < U; ++uu) {
#pragma unroll
            for (int off = LPG / 2; off > 0; off >>= 1) part[uu] += __shfl_xor_sync(FULL, part[uu], off);
          }
#pragma unroll
          for (int uu = 0; uu < U; ++uu) {
            const int j = base + uu * G + g;
            const float v = __int_as_float(__shfl_sync(FULL, my.y, j & 31));
            const int o = __shfl_sync(FULL, myo, j & 31);
            if (lg == 0 && j < b) {
              float res = v * part[uu];
              if (k0 > 0) res += out[o];
              out[o] = res;
            }
          }
        }
      }
    }
  };
  auto pass_end = [&](int) {};
  const StageLayout L{TW * KCP, TS, true, kSddmmStages};
  dense_pipeline<kBulk>(u, vtiles, dense_cols, trp, ent, d_oidx, Y, ldy, K, KCP, L, smem, full, empty, body,
                        pass_end);
}

// ------------------------------------------------------------------ host dispatch
inline int next_pow2(int x) {
  int p = 1;
  while (p < x) p <<= 1;
  return p;
}

constexpr int kSparseWarps = 8;

template <int LPG, int VEC>
int run_spmm(sr_csr_s* h, const float* B, int64_t K, int64_t ldb, float* C, int64_t ldc,
             cudaStream_t s, int32_t* launches) {
  DevPlan& P = h->plan;
  constexpr int KC = LPG * VEC;
  constexpr int U = (LPG == 32) ? 8 : 4;  // gathers in flight per lane (phase S)
  constexpr int UD = 4;                   // shared-memory reads in flight per lane (phase D)
  if (P.n_units > 0) {
    const int TW = P.tile_cols;
    const size_t smem = (size_t)kSpmmStages * StageLayout{TW * KC, P.trp_stride, false, kSpmmStages}.bytes() + kUnitColsBytes;
    if (P.n_dslots > 0 && P.dscratch_k < K) {
      SR_TRY(P.dscratch.alloc((size_t)P.n_dslots * P.panel_rows * K));
      P.dscratch_k = K;
    }
    auto launch = [&](auto kern) -> int {
      SR_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      kern<<<(unsigned)P.n_units, (kDenseWarps + 1) * 32, smem, s>>>(
          P.units.p, P.vtiles.p, P.dense_cols.p, P.trp.p, P.d_ent.p, P.drow_ptr.p, P.pos_out.p, B, ldb, C, ldc,
          (int)K, TW, P.trp_stride, P.panel_rows, P.dscratch.p, P.dsplit_info.p, P.dsplit_counter.p);
      SR_CUDA_TRY(cudaGetLastError());
      return SR_OK;
    };
    if (P.profiling) SR_TRY(prof_begin(P, 1, s));
    if (VEC == 4) {
      if (P.panel_rows <= 8 * kDenseWarps) SR_TRY(launch(spmm_dense_kernel<LPG, VEC, UD, 8, true>));
      else SR_TRY(launch(spmm_dense_kernel<LPG, VEC, UD, 16, true>));
    } else {
      SR_TRY(launch(spmm_dense_kernel<LPG, VEC, UD, 16, false>));
    }
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
    spmm_sparse_kernel<LPG, VEC, U><<<grid, kSparseWarps * 32, 0, s>>>(
        P.items.p, P.item_meta.p, P.n_items, P.s_ent.p, B, ldb, C, ldc, (int)K, P.scratch.p,
        P.split_info.p, P.split_counter.p);
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
  if (P.n_units > 0) {
    const int TW = P.tile_cols;
    const size_t smem = (size_t)kSddmmStages * StageLayout{TW * NCH_D * KC, P.trp_stride, true, kSddmmStages}.bytes() + kUnitColsBytes;
    auto launch = [&](auto kern) -> int {
      SR_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      kern<<<(unsigned)P.n_units, (kDenseWarps + 1) * 32, smem, s>>>(
          P.units.p, P.vtiles.p, P.dense_cols.p, P.trp.p, P.d_ent.p, P.d_oidx.p, P.pos_xrow.p, X, ldx, Y, ldy,
          (int)K, TW, P.trp_stride, out);
      SR_CUDA_TRY(cudaGetLastError());
      return SR_OK;
    };
    constexpr int UD = 4;
    if (P.profiling) SR_TRY(prof_begin(P, 3, s));
    if (VEC == 4) {
      if (P.panel_rows <= 8 * kDenseWarps) SR_TRY(launch(sddmm_dense_kernel<LPG, VEC, UD, NCH_D, 8, true>));
      else SR_TRY(launch(sddmm_dense_kernel<LPG, VEC, UD, NCH_D, 16, true>));
    } else {
      SR_TRY(launch(sddmm_dense_kernel<LPG, VEC, UD, NCH_D, 16, false>));
    }
    if (P.profiling) SR_TRY(prof_end(P, s));
    ++*launches;
  }
  if (P.n_sitems > 0) {
    const unsigned grid = (unsigned)((P.n_sitems + kSparseWarps - 1) / kSparseWarps);
    if (P.profiling) SR_TRY(prof_begin(P, 4, s));
    sddmm_sparse_kernel<LPG, VEC, U, NCH><<<grid, kSparseWarps * 32, 0, s>>>(
        P.items.p, P.n_sitems, P.s_ent.p, P.s_oidx.p, X, ldx, Y, ldy, (int)K, out);
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
}  // namespace

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
