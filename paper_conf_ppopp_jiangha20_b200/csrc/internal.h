// Internal declarations of libsr (the product library).  Shares nothing with oracle/.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <memory>
#include <utility>
#include <vector>

#include "../../include/sr.h"

namespace sr {

void set_error(const std::string& msg);

struct Status {
  int code = SR_OK;
  static Status ok() { return Status(); }
};

#define SR_CUDA_TRY(expr)                                                              \
  do {                                                                                 \
    cudaError_t _e = (expr);                                                           \
    if (_e != cudaSuccess) {                                                           \
      ::sr::set_error(std::string(#expr) + ": " + cudaGetErrorString(_e));             \
      return SR_ECUDA;                                                                 \
    }                                                                                  \
  } while (0)

#define SR_TRY(expr)        \
  do {                      \
    int _rc = (expr);       \
    if (_rc != SR_OK) return _rc; \
  } while (0)

// RAII device buffer
// Stream-ordered pool allocations (cudaMallocAsync) for the reorder's temporaries: the two LSH
// rounds allocate and free GBs of sort buffers; the device's default pool keeps them mapped
// between rounds instead of a cudaMalloc / cudaFree of each (sr_reorder trims it at the end).
void keep_pool_memory();

template <typename T>
struct DevBuf {
  T* p = nullptr;
  size_t n = 0;
  cudaStream_t pool = nullptr;  // non-null: stream-ordered allocation on this stream
  DevBuf() = default;
  explicit DevBuf(cudaStream_t s) : pool(s) { keep_pool_memory(); }
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  DevBuf(DevBuf&& o) noexcept : p(o.p), n(o.n), pool(o.pool) { o.p = nullptr; o.n = 0; }
  DevBuf& operator=(DevBuf&& o) noexcept {
    if (this != &o) {
      release();
      p = o.p;
      n = o.n;
      pool = o.pool;
      o.p = nullptr;
      o.n = 0;
    }
    return *this;
  }
  ~DevBuf() { release(); }
  void release() {
    if (p) {
      if (pool)
        cudaFreeAsync(p, pool);
      else
        cudaFree(p);
    }
    p = nullptr;
    n = 0;
  }
  int alloc(size_t count) {
    release();
    if (count == 0) count = 1;
    const cudaError_t e = pool ? cudaMallocAsync(reinterpret_cast<void**>(&p), count * sizeof(T), pool)
                               : cudaMalloc(&p, count * sizeof(T));
    if (e != cudaSuccess) {
      cudaGetLastError();
      set_error("cudaMalloc of " + std::to_string(count * sizeof(T)) + " bytes failed");
      p = nullptr;
      return SR_ENOMEM;
    }
    n = count;
    return SR_OK;
  }
  int upload(const T* host, size_t count, cudaStream_t s) {  // n = count (0 allowed)
    SR_TRY(alloc(count));
    n = count;
    if (count) SR_CUDA_TRY(cudaMemcpyAsync(p, host, count * sizeof(T), cudaMemcpyHostToDevice, s));
    return SR_OK;
  }
  int upload(const std::vector<T>& v, cudaStream_t s) { return upload(v.data(), v.size(), s); }
};

// A column-sorted CSR on the host (canonical form of the caller's matrix).
struct HostCSR {
  int64_t M = 0, N = 0;
  std::vector<int64_t> rowptr;  // M+1
  std::vector<int32_t> col;     // nnz
  std::vector<float> val;       // nnz
  std::vector<int32_t> opos;    // nnz: caller's original index of each canonical nnz
  bool identity_pos = true;
  int64_t nnz() const { return rowptr.empty() ? 0 : rowptr.back(); }
};

// ASpT tiling of a row order (host result, positions q = index into perm).
struct Tiling {
  int64_t npanels = 0;
  std::vector<int64_t> dense_ptr;   // npanels+1
  std::vector<int32_t> dense_cols;  // Σ|D_p|
  std::vector<int64_t> drow_ptr;    // M+1 over positions
  std::vector<int32_t> d_slot;      // dense nnz: slot in D_p (ascending per position)
  std::vector<int64_t> d_cidx;      // dense nnz: canonical nnz index
  std::vector<int64_t> rrow_ptr;    // M+1 over positions
  std::vector<int32_t> r_col;       // remainder nnz: column (CSR order)
  std::vector<int64_t> r_cidx;      // remainder nnz: canonical nnz index
  int64_t n_dense() const { return drow_ptr.empty() ? 0 : drow_ptr.back(); }
};

// Phase-S work item: one warp processes entries [e0, e1) of the remainder stream.
struct __align__(16) Item {
  int32_t e0, e1;
  int32_t xrow;  // original row id (X row for SDDMM)
  int32_t out;   // SpMM output row (original id, or packed shard index)
};

// The phase-S entry streams carry kEntPad trailing padding entries ({0, 0}, output index -1) so
// a kernel may load entries in pairs past the end of its last task.
constexpr int kEntPad = 8;

constexpr uint32_t kItemRMW = 1u << 31;    // C[out] += partial (row also has dense-tile nnz)
constexpr uint32_t kItemSplit = 1u << 30;  // partial of a split long row -> scratch slot
constexpr uint32_t kItemSlotMask = (1u << 30) - 1;

// Phase-D execution tile: <= kMaxExecTile dense columns of one panel and (a row subset of)
// their entries; its entry block is 16-byte aligned so one bulk copy stages it.
struct __align__(16) VTile {
  int32_t ent0;   // first entry in d_ent / d_oidx (multiple of 4)
  int32_t nent;   // entries in the block, padded to a multiple of 4
  int32_t col0;   // dense_cols index of the first staged column
  int32_t ncols;  // staged columns
};
// Phase-D work unit (one CTA): up to kMaxUnitTiles consecutive virtual tiles of one panel.
struct __align__(16) DUnit {
  int32_t q0, nrows;  // panel positions [q0, q0+nrows)
  int32_t vt0, nvt;   // virtual tiles [vt0, vt0+nvt)
  int32_t split;      // -1: the unit covers its whole panel; else its partial-sum slot
  int32_t pad0, pad1, pad2;
};
constexpr int kRtMaxRows = 8;                        // register-tile engine: panel rows
constexpr int64_t kRtChunk = 1024;                   // register-tile stream entries per warp (chunk)
constexpr int32_t kRtHeader = (int32_t)0x80000000u;  // marks a column header entry
constexpr int kMaxUnitTiles = 32;  // one VTile per producer lane; whole panels of <= 2048 dense
                                   // columns are one unit (no split partials / combine)
constexpr int kMaxExecTile = 64;
constexpr int kMaxTileEntries = 384;  // SpMM: 3 stages + blob ring must fit twice per SM
// producer-side record of a unit: DUnit and its VTiles (16-byte aligned)
constexpr int kMaxUnitBlobBytes = 32 + kMaxUnitTiles * 16;

struct TmapKey {
  const void* base = nullptr;
  int64_t rows = 0, K = 0, ld = 0;
  int box = 0;
  bool operator==(const TmapKey& o) const {
    return base == o.base && rows == o.rows && K == o.K && ld == o.ld && box == o.box;
  }
};

// Device-resident execution plan.
struct DevPlan {
  // cached TMA tensor map of the last phase-D operand (exec.cu: cached_row_gather_map)
  alignas(64) unsigned char tmap_bytes[128] = {};
  TmapKey tmap_key;
  bool tmap_valid = false, tmap_ok = false;
  // phase D
  DevBuf<DUnit> units;
  int64_t n_units = 0;
  DevBuf<int32_t> dense_cols;
  DevBuf<VTile> vtiles;
  DevBuf<int4> blobs;         // per unit: DUnit | VTile[nvt] | dense column ids (16-byte records)
  DevBuf<int2> blob_meta;     // per unit: {offset in 16-byte words, bytes}
  DevBuf<int32_t> trp;        // per virtual tile: trp_stride offsets relative to its entry block
  int32_t trp_stride = 68;
  DevBuf<int32_t> drow_ptr;   // positions -> dense nnz offsets (only "row has dense nnz" is used)
  DevBuf<int2> d_ent;         // tile-major {slot in tile, __float_as_int(val)}
  DevBuf<int32_t> d_oidx;     // SDDMM output index per dense nnz (tile-major)
  DevBuf<int2> dsplit_info;   // per split unit: {first slot, nchunks}
  DevBuf<int32_t> dsplit_counter;
  int64_t n_dslots = 0;
  DevBuf<float> dscratch;     // n_dslots × panel_rows × dscratch_k
  int64_t dscratch_k = 0;
  // phase D, register-tile engine (panels of <= kRtMaxRows rows; api.cpp: build_rt_stream)
  int64_t n_rt = 0;
  DevBuf<int4> rt_units;      // one warp per panel: {e0, e1, first position, rows}
  DevBuf<int2> rt_ent;        // column headers {col | kRtHeader, row mask} + {row, value bits}
  DevBuf<int32_t> rt_oidx;    // SDDMM output index per value entry (-1: header / padding)
  DevBuf<int2> rt_split;      // per unit: {panel's first slot, chunk << 16 | chunks} ({-1, 1}: whole panel)
  DevBuf<int32_t> rt_counter; // per split panel (its first slot): finished chunks
  int64_t n_rt_slots = 0;
  DevBuf<float> rt_scratch;   // n_rt_slots × kRtMaxRows × rt_scratch_k partial sums
  int64_t rt_scratch_k = 0;
  DevBuf<int32_t> pos_xrow;   // position -> original row
  DevBuf<int32_t> pos_out;    // position -> SpMM output row
  DevBuf<int32_t> dense_out;  // position -> SpMM output row if the row has dense nnz, else -1
  // phase S
  DevBuf<int2> s_ent;         // {col, __float_as_int(val)} remainder stream
  DevBuf<int32_t> s_oidx;     // SDDMM output index per remainder nnz
  DevBuf<Item> items;         // SpMM items (remainder rows, split chunks, zero rows)
  DevBuf<uint32_t> item_meta;
  int64_t n_items = 0;
  DevBuf<int4> tasks;         // SpMM row-group tasks {e0, e1, first item, end item} (build_tasks)
  int64_t n_tasks = 0;
  DevBuf<int4> stasks;        // SDDMM row-group tasks (<= 8 rows each, non-empty rows only)
  DevBuf<int32_t> task_ticket;  // [0] SpMM, [1] SDDMM task kernels' work counters (exec.cu: first_ticket)
  int64_t n_stasks = 0;
  DevBuf<Item> sitems;        // SDDMM items (remainder rows / chunks only)
  int64_t n_sitems = 0;
  DevBuf<int2> split_info;    // per scratch slot: {first slot, nchunks}
  DevBuf<int32_t> split_counter;
  int64_t n_slots = 0;
  DevBuf<float> scratch;      // n_slots × scratch_k
  int64_t scratch_k = 0;
  int32_t tile_cols = 64;
  int32_t panel_rows = 64;
  int64_t max_dense_per_panel = 0;
  sr_traffic_model traffic{};
  // profiling (sr_set_profiling)
  bool profiling = false;
  cudaEvent_t ev[8] = {};
  int32_t kinds[4] = {};
  int32_t nrec = 0;
};

// profiling helpers (exec.cu)
int prof_begin(DevPlan& P, int kind, cudaStream_t s);
int prof_end(DevPlan& P, cudaStream_t s);

}  // namespace sr

struct sr_csr_s {
  int device = 0;
  sr::HostCSR A;
  bool reordered = false;
  bool identity_ready = false;  // the identity plan has been built (ensure_plan)
  sr_reorder_params params{};
  std::vector<int32_t> perm1, perm2;
  sr::Tiling tiles;
  sr_plan_stats stats{};
  std::vector<int32_t> shard_rows;
  std::vector<int64_t> shard_nnz_ids;
  sr::DevPlan plan;
  int32_t last_launches = 0;
  cudaStream_t init_stream = nullptr;
};

namespace sr {
// tiler.cpp
void tile_rows(const HostCSR& A, const std::vector<int32_t>& perm, int32_t panel_rows,
               int32_t dense_min, Tiling& t);
void avgsim_positions(const Tiling& t, uint64_t* num, uint64_t* den);
int64_t dense_count(const HostCSR& A, const std::vector<int32_t>& perm, int32_t panel_rows, int32_t dense_min);
// cluster.cpp
void cluster_rows(int64_t M, const int64_t* rowptr, const int32_t* col, int64_t npairs,
                  const uint64_t* pairs, const uint32_t* inter, const uint32_t* uni,
                  int32_t threshold_size, int32_t* perm, const uint64_t* pairs_by_key = nullptr);
void partition_panels(int64_t npanels, const int64_t* w, int32_t G, int64_t* cuts);
// Host vector whose resize() leaves new elements uninitialised (a D2H copy overwrites them).
template <class T>
struct DefaultInitAlloc : std::allocator<T> {
  template <class U>
  struct rebind {
    using other = DefaultInitAlloc<U>;
  };
  DefaultInitAlloc() = default;
  template <class U>
  DefaultInitAlloc(const DefaultInitAlloc<U>&) noexcept {}
  template <class U>
  void construct(U* p) noexcept {
    ::new (static_cast<void*>(p)) U;
  }
  template <class U, class... A>
  void construct(U* p, A&&... a) {
    ::new (static_cast<void*>(p)) U(std::forward<A>(a)...);
  }
};
template <class T>
using HostVec = std::vector<T, DefaultInitAlloc<T>>;
// Device -> pageable host copy through a pinned two-chunk staging ring, the chunk copies out of
// the ring done by all host threads (first touch of the destination pages included); synchronous.
int d2h_staged(void* dst, const void* src, size_t bytes, cudaStream_t s);
// lsh.cu : device LSH candidate generation + exact Jaccard (sorted J order).
// Returns candidate pairs sorted by (J desc, pair asc) with their (inter, uni).
int lsh_candidates(const int64_t* rowptr_h, const int32_t* col_h, int64_t M, int64_t nnz,
                   const sr_reorder_params& p, cudaStream_t s, HostVec<uint64_t>& pairs_by_j,
                   HostVec<uint32_t>& inter, HostVec<uint32_t>& uni, int64_t* E,
                   HostVec<uint64_t>* pairs_by_key = nullptr);
// exec.cu : launchers
int launch_spmm(sr_csr_s* h, const float* B, int64_t K, int64_t ldb, float* C, int64_t ldc,
                cudaStream_t s, int32_t* launches);
int launch_sddmm(sr_csr_s* h, const float* X, int64_t ldx, const float* Y, int64_t ldy, int64_t K,
                 float* out, cudaStream_t s, int32_t* launches);
int launch_scatter_rows(const float* src, int64_t lds, const int32_t* rows, int64_t n, int64_t K, float* dst,
                        int64_t ldd, cudaStream_t s);
int launch_scatter_values(const float* src, const int64_t* ids, int64_t n, float* dst, cudaStream_t s);
int launch_set_values(int2* ent, const int32_t* oidx, int64_t n, const float* vals, cudaStream_t s);
}  // namespace sr
