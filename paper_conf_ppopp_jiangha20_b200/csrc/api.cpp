// C ABI of libsr (include/sr.h): ingest, the reorder driver (Fig 5 workflow, P:137;
// decision rules P:265), plan construction, metadata export, host entry points.
#include <algorithm>
#include <array>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <string>
#include <vector>

#ifdef _OPENMP
#include <omp.h>
#endif

#include "internal.h"

namespace sr {

static thread_local std::string g_err;
void set_error(const std::string& msg) { g_err = msg; }

void keep_pool_memory() {
  static int done = [] {
    int dev = 0;
    cudaMemPool_t pool;
    if (cudaGetDevice(&dev) == cudaSuccess && cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
      uint64_t thr = ~0ull;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    cudaGetLastError();
    return 1;
  }();
  (void)done;
}

static void trim_pool(int device) {
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) cudaMemPoolTrimTo(pool, 0);
  cudaGetLastError();
}


namespace {

constexpr int32_t kSplitChunk = 256;  // phase-S work item: at most this many nnz

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

double now_s() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int einval(const std::string& m) {
  set_error(m);
  return SR_EINVAL;
}

// Items of phase S for a sequence of (position-ordered) rows.
struct ItemBuilder {
  std::vector<Item> items;
  std::vector<uint32_t> meta;
  std::vector<int2> split_info;  // per slot
  int64_t n_slots = 0;
  void add_row(int32_t e0, int32_t e1, int32_t xrow, int32_t out, bool rmw) {
    const int32_t len = e1 - e0;
    if (len <= kSplitChunk) {
      items.push_back(Item{e0, e1, xrow, out});
      meta.push_back(rmw ? kItemRMW : 0u);
      return;
    }
    const int32_t nch = (len + kSplitChunk - 1) / kSplitChunk;
    const int32_t first = (int32_t)n_slots;
    for (int32_t c = 0; c < nch; ++c) {
      const int32_t a = e0 + c * kSplitChunk, b = std::min(e1, a + kSplitChunk);
      items.push_back(Item{a, b, xrow, out});
      meta.push_back((rmw ? kItemRMW : 0u) | kItemSplit | (uint32_t)(first + c));
      split_info.push_back(make_int2(first, nch));
    }
    n_slots += nch;
  }
};

// Bytes model of phase S: entries of consecutive groups of 8 items (one CTA) that share a
// column load it once (access model O14 / P:111); distinct columns = compulsory.
void sparse_traffic(const ItemBuilder& ib, int64_t n_nonzero, int64_t n_zero, const std::vector<int2>& ent,
                    int64_t N, sr_traffic_model& t) {
  std::vector<uint8_t> seen((size_t)N, 0);
  int64_t loads = 0, nnz = 0, rows = 0;
  const int64_t ngroups = (n_nonzero + 7) / 8;
#pragma omp parallel reduction(+ : loads, nnz, rows)
  {
    std::vector<int32_t> cols;
#pragma omp for schedule(dynamic, 1024)
    for (int64_t grp = 0; grp < ngroups; ++grp) {
      cols.clear();
      for (int64_t it = grp * 8; it < std::min(n_nonzero, grp * 8 + 8); ++it) {
        const Item& x = ib.items[it];
        nnz += x.e1 - x.e0;
        const uint32_t m = ib.meta[it];
        if (!(m & kItemSplit) || (m & kItemSlotMask) == (uint32_t)ib.split_info[m & kItemSlotMask].x) ++rows;
        for (int32_t e = x.e0; e < x.e1; ++e) {
          cols.push_back(ent[e].x);
          __atomic_store_n(&seen[ent[e].x], (uint8_t)1, __ATOMIC_RELAXED);
        }
      }
      std::sort(cols.begin(), cols.end());
      loads += std::unique(cols.begin(), cols.end()) - cols.begin();
    }
  }
  int64_t distinct = 0;
#pragma omp parallel for reduction(+ : distinct) schedule(static)
  for (int64_t c = 0; c < N; ++c) distinct += seen[c];
  t.sparse_nnz = nnz;
  t.sparse_items = n_nonzero + n_zero;
  t.sparse_rows = rows;
  t.zero_rows = n_zero;
  t.sparse_group_loads = loads;
  t.sparse_distinct_cols = distinct;
}

// Row-group tasks of the SpMM phase-S kernel (exec.cu: spmm_task_kernel): greedy runs of
// consecutive items, at most 32 items and task_nnz entries (a longer item stands alone; a
// split chunk always stands alone), whose items are contiguous in the entry stream; a task holds
// either only non-empty rows or only zero rows.
int32_t task_nnz() {
  static const int32_t v = [] {
    const char* e = getenv("SR_TASK_NNZ");
    const int x = e ? atoi(e) : 256;  // measured best of 64..1024 on C2 (profiles/r01/tasknnz, NOTES.md)
    return x < 1 ? 1 : x;
  }();
  return v;
}

std::vector<int4> build_tasks(const ItemBuilder& ib, int64_t n, int64_t max_rows) {
  std::vector<int4> tasks;
  const int32_t T = task_nnz();
  int64_t i = 0;
  while (i < n) {
    const int64_t start = i;
    int32_t e0 = -1, e1 = -1;
    if (ib.meta[i] & kItemSplit) {
      e0 = ib.items[i].e0;
      e1 = ib.items[i].e1;
      ++i;
    } else {
      int32_t tot = 0;
      const bool zero = ib.items[i].e1 == ib.items[i].e0;
      while (i < n && i - start < max_rows && !(ib.meta[i] & kItemSplit)) {
        const Item& x = ib.items[i];
        const int32_t len = x.e1 - x.e0;
        if ((len == 0) != zero) break;  // zero rows and non-empty rows go to separate tasks
        if (len > 0) {
          if (e0 >= 0 && (x.e0 != e1 || tot + len > T)) break;
          if (e0 < 0) e0 = e1 = x.e0;
          e1 += len;
          tot += len;
        }
        ++i;
      }
      if (e0 < 0) e0 = e1 = 0;
    }
    tasks.push_back(make_int4(e0, e1, (int32_t)start, (int32_t)i));
  }
  return tasks;
}

int upload_items(DevPlan& P, ItemBuilder& ib, int64_t n_sddmm_items, cudaStream_t s) {
  const std::vector<int4> tasks = build_tasks(ib, (int64_t)ib.items.size(), 32);
  P.n_tasks = (int64_t)tasks.size();
  SR_TRY(P.tasks.upload(tasks, s));
  // SDDMM: the non-empty items only (a prefix), at most 8 rows per task (X rows staged in smem)
  const std::vector<int4> stasks = build_tasks(ib, n_sddmm_items, 8);
  P.n_stasks = (int64_t)stasks.size();
  SR_TRY(P.stasks.upload(stasks, s));
  SR_TRY(P.task_ticket.alloc(2));
  SR_CUDA_TRY(cudaMemsetAsync(P.task_ticket.p, 0, 2 * sizeof(int32_t), s));
  P.n_items = (int64_t)ib.items.size();
  P.n_sitems = n_sddmm_items;
  SR_TRY(P.items.upload(ib.items, s));
  SR_TRY(P.item_meta.upload(ib.meta, s));
  P.n_slots = ib.n_slots;
  if (ib.n_slots > 0) {
    SR_TRY(P.split_info.upload(ib.split_info, s));
    SR_TRY(P.split_counter.alloc((size_t)ib.n_slots));
    SR_CUDA_TRY(cudaMemsetAsync(P.split_counter.p, 0, ib.n_slots * sizeof(int32_t), s));
  }
  P.scratch.release();
  P.scratch_k = 0;
  return SR_OK;
}

// Identity plan: plain row-wise kernels over the canonical CSR.
int build_identity_plan(sr_csr_s* h, cudaStream_t s) {
  const HostCSR& A = h->A;
  DevPlan& P = h->plan;
  const int64_t nnz = A.nnz();
  std::vector<int2> ent((size_t)nnz);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < nnz; ++e) {
    ent[e].x = A.col[e];
    ent[e].y = *reinterpret_cast<const int32_t*>(&A.val[e]);
  }
  std::vector<int32_t> o((size_t)nnz);
  if (A.identity_pos)
    std::iota(o.begin(), o.end(), 0);
  else
    std::copy(A.opos.begin(), A.opos.end(), o.begin());
  ent.resize((size_t)nnz + kEntPad, make_int2(0, 0));
  o.resize((size_t)nnz + kEntPad, -1);
  SR_TRY(P.s_oidx.upload(o, s));
  ItemBuilder ib;
  std::vector<int32_t> zero_rows;
  for (int64_t r = 0; r < A.M; ++r) {
    if (A.rowptr[r + 1] > A.rowptr[r])
      ib.add_row((int32_t)A.rowptr[r], (int32_t)A.rowptr[r + 1], (int32_t)r, (int32_t)r, false);
    else
      zero_rows.push_back((int32_t)r);
  }
  const int64_t n_nonzero = (int64_t)ib.items.size();
  for (int32_t r : zero_rows) {
    ib.items.push_back(Item{0, 0, r, r});
    ib.meta.push_back(0u);
  }
  std::memset(&P.traffic, 0, sizeof(P.traffic));
  sparse_traffic(ib, n_nonzero, (int64_t)zero_rows.size(), ent, A.N, P.traffic);
  SR_TRY(P.s_ent.upload(ent, s));
  SR_TRY(upload_items(P, ib, n_nonzero, s));
  P.n_units = 0;
  SR_CUDA_TRY(cudaStreamSynchronize(s));
  return SR_OK;
}

// Register-tile stream of the dense nnz (panels of <= kRtMaxRows rows, exec.cu:
// spmm_rtile_kernel / sddmm_rtile_kernel).  Per panel, its dense columns in slot order (count
// desc, column asc: R18); per column one header entry {col | kRtHeader, mask of the panel rows
// holding it} followed by one {row, value bits} entry per such row, rows ascending.  A column's
// entries never straddle a 32-entry batch of its panel (padding entries {0, 0} in between), so
// a warp decodes each batch on its own.  Units (one warp per panel) are ordered largest first.
int build_rt_stream(sr_csr_s* h, int64_t pb, int64_t pe, const std::vector<int32_t>& d_out, DevPlan& P,
                    cudaStream_t s) {
  const HostCSR& A = h->A;
  const Tiling& T = h->tiles;
  const int64_t M = A.M;
  const int32_t PR = h->params.panel_rows;
  std::vector<int2> ent;
  std::vector<int32_t> oidx;
  std::vector<int4> units;
  std::vector<std::array<int32_t, 3>> cell;  // (slot, row, dense nnz index)
  std::vector<int2> split;                   // per unit: {panel's first slot, chunk << 16 | chunks}
  int64_t n_slots = 0;
  for (int64_t p = pb; p < pe; ++p) {
    const int64_t dc0 = T.dense_ptr[p], dc1 = T.dense_ptr[p + 1];
    if (dc1 == dc0) continue;
    const int64_t q0 = p * PR, nrows = std::min<int64_t>(M, q0 + PR) - q0;
    cell.clear();
    for (int64_t r = 0; r < nrows; ++r)
      for (int64_t e = T.drow_ptr[q0 + r]; e < T.drow_ptr[q0 + r + 1]; ++e)
        cell.push_back({T.d_slot[e], (int32_t)r, (int32_t)e});
    std::sort(cell.begin(), cell.end());
    // a panel with more than kRtChunk entries is cut at column boundaries into chunks, one warp
    // each; SpMM chunks leave partial sums and the last one adds them in chunk order
    int64_t e0 = (int64_t)ent.size();
    const size_t first_unit = units.size();
    size_t i = 0;
    while (i < cell.size()) {
      size_t j = i;
      uint32_t mask = 0;
      while (j < cell.size() && cell[j][0] == cell[i][0]) mask |= 1u << cell[j++][1];
      const int64_t len = 1 + (int64_t)(j - i);
      int64_t at = ((int64_t)ent.size() - e0) % 32;
      if ((int64_t)ent.size() - e0 + (at + len > 32 ? 32 - at : 0) + len > kRtChunk) {  // close the chunk
        units.push_back(make_int4((int32_t)e0, (int32_t)ent.size(), (int32_t)q0, (int32_t)nrows));
        e0 = (int64_t)ent.size();
        at = 0;
      }
      if (at + len > 32)  // keep the column inside one 32-entry batch
        for (int64_t k = at; k < 32; ++k) {
          ent.push_back(make_int2(0, 0));
          oidx.push_back(-1);
        }
      ent.push_back(make_int2((int32_t)(T.dense_cols[dc0 + cell[i][0]] | kRtHeader), (int32_t)mask));
      oidx.push_back(-1);
      for (size_t k = i; k < j; ++k) {
        const int64_t e = cell[k][2];
        ent.push_back(make_int2(cell[k][1], *reinterpret_cast<const int32_t*>(&A.val[T.d_cidx[e]])));
        oidx.push_back(d_out[e]);
      }
      i = j;
    }
    units.push_back(make_int4((int32_t)e0, (int32_t)ent.size(), (int32_t)q0, (int32_t)nrows));
    const int32_t nch = (int32_t)(units.size() - first_unit);
    for (int32_t c = 0; c < nch; ++c)
      split.push_back(nch > 1 ? make_int2((int32_t)n_slots, (c << 16) | nch) : make_int2(-1, 1));
    if (nch > 1) n_slots += nch;
  }
  {  // largest first (balance); the split records travel with their units
    std::vector<size_t> ord(units.size());
    std::iota(ord.begin(), ord.end(), 0);
    std::stable_sort(ord.begin(), ord.end(), [&](size_t x, size_t y) {
      return units[x].y - units[x].x > units[y].y - units[y].x;
    });
    std::vector<int4> u2(units.size());
    std::vector<int2> s2(units.size());
    for (size_t k = 0; k < ord.size(); ++k) {
      u2[k] = units[ord[k]];
      s2[k] = split[ord[k]];
    }
    units.swap(u2);
    split.swap(s2);
  }
  ent.resize(ent.size() + kEntPad, make_int2(0, 0));
  oidx.resize(oidx.size() + kEntPad, -1);
  P.n_rt = (int64_t)units.size();
  P.n_rt_slots = n_slots;
  SR_TRY(P.rt_split.upload(split, s));
  if (n_slots > 0) {
    SR_TRY(P.rt_counter.alloc((size_t)n_slots));
    SR_CUDA_TRY(cudaMemsetAsync(P.rt_counter.p, 0, n_slots * sizeof(int32_t), s));
  }
  SR_TRY(P.rt_units.upload(units, s));
  SR_TRY(P.rt_ent.upload(ent, s));
  SR_TRY(P.rt_oidx.upload(oidx, s));
  return SR_OK;
}

// The identity plan on first use of a handle without a reordered plan.  Synchronous (once).
int ensure_plan(sr_csr_s* h) {
  if (h->reordered || h->identity_ready) return SR_OK;
  SR_TRY(build_identity_plan(h, h->init_stream));
  h->identity_ready = true;
  return SR_OK;
}

// Device plan of a (possibly sharded) tiling.  Built into fresh buffers and installed only when
// every upload and the final synchronisation succeeded, so a failure (ENOMEM, a CUDA error)
// leaves the handle's previous plan intact.
int build_exec_plan_into(sr_csr_s* h, int64_t pb, int64_t pe, cudaStream_t s, DevPlan& P,
                         std::vector<int32_t>& shard_rows, std::vector<int64_t>& shard_nnz_ids);

int build_exec_plan(sr_csr_s* h, int64_t pb, int64_t pe, cudaStream_t s) {
  DevPlan P;
  std::vector<int32_t> rows;
  std::vector<int64_t> ids;
  const int rc = build_exec_plan_into(h, pb, pe, s, P, rows, ids);
  if (rc != SR_OK) {
    cudaStreamSynchronize(s);  // no copy into P's buffers may still be in flight when they are freed
    cudaGetLastError();
    return rc;
  }
  for (int i = 0; i < 8; ++i) {  // the profiling events belong to the handle
    P.ev[i] = h->plan.ev[i];
    h->plan.ev[i] = nullptr;
  }
  P.profiling = h->plan.profiling;
  h->plan = std::move(P);
  h->shard_rows = std::move(rows);
  h->shard_nnz_ids = std::move(ids);
  return SR_OK;
}

int build_exec_plan_into(sr_csr_s* h, int64_t pb, int64_t pe, cudaStream_t s, DevPlan& P,
                         std::vector<int32_t>& shard_rows, std::vector<int64_t>& shard_nnz_ids) {
  const HostCSR& A = h->A;
  const Tiling& T = h->tiles;
  const int64_t M = A.M;
  const int32_t PR = h->params.panel_rows;
  const bool sharded = h->params.world > 1;
  const int64_t q0s = std::min<int64_t>(M, pb * PR), q1s = std::min<int64_t>(M, pe * PR);
  const std::vector<int32_t>& perm1 = h->perm1;
  // shard rows / packed nnz order: by position, dense (slot order) then remainder (CSR order)
  shard_rows.assign(perm1.begin() + q0s, perm1.begin() + q1s);
  std::vector<int32_t> d_out((size_t)T.n_dense(), 0), r_out(T.r_col.size(), 0);
  shard_nnz_ids.clear();
  if (!sharded) {  // outputs in the caller's order: every index is the caller's own position
    const int64_t nd = T.n_dense(), nr = (int64_t)T.r_col.size();
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < nd; ++e) d_out[e] = (int32_t)(A.identity_pos ? T.d_cidx[e] : A.opos[T.d_cidx[e]]);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < nr; ++e) r_out[e] = (int32_t)(A.identity_pos ? T.r_cidx[e] : A.opos[T.r_cidx[e]]);
    shard_nnz_ids.resize((size_t)(nd + nr));
  } else {
    int64_t k = 0;
    for (int64_t q = q0s; q < q1s; ++q) {
      for (int64_t e = T.drow_ptr[q]; e < T.drow_ptr[q + 1]; ++e) {
        const int64_t orig = A.identity_pos ? T.d_cidx[e] : A.opos[T.d_cidx[e]];
        d_out[e] = (int32_t)(sharded ? k : orig);
        shard_nnz_ids.push_back(orig);
        ++k;
      }
      for (int64_t e = T.rrow_ptr[q]; e < T.rrow_ptr[q + 1]; ++e) {
        const int64_t orig = A.identity_pos ? T.r_cidx[e] : A.opos[T.r_cidx[e]];
        r_out[e] = (int32_t)(sharded ? k : orig);
        shard_nnz_ids.push_back(orig);
        ++k;
      }
    }
  }
  if (!sharded) {  // single shard: outputs come back in the caller's order
    std::iota(shard_rows.begin(), shard_rows.end(), 0);
    std::iota(shard_nnz_ids.begin(), shard_nnz_ids.end(), 0);
  }
  // phase D: execution tiles of <= kMaxExecTile dense columns (the plan's tiles of tile_cols
  // columns are reported in the metadata and staged in sub-tiles); each tile's entries are
  // stored tile-major with panel-row offsets (trp) relative to the tile's entry block; a
  // tile with more than kMaxTileEntries entries is split by rows into virtual tiles that
  // stage the same columns; units of <= kMaxUnitTiles virtual tiles (giant panels -> split
  // units with an ordered combine).
  const int32_t TW = std::min(h->params.tile_cols, kMaxExecTile);
  const int32_t TS = (PR + 1 + 3) / 4 * 4;
  std::vector<DUnit> units;
  std::vector<VTile> vtiles;
  std::vector<int2> dsplit;
  std::vector<int32_t> trp;
  std::vector<int2> de;
  std::vector<int32_t> deo;
  de.reserve((size_t)T.n_dense() + T.n_dense() / 4);
  deo.reserve((size_t)T.n_dense() + T.n_dense() / 4);
  int64_t maxd = 0, n_dslots = 0;
  std::vector<int64_t> cur((size_t)PR), stop((size_t)PR);
  auto pad4 = [&]() {
    while (de.size() % 4) {
      de.push_back(make_int2(0, 0));
      deo.push_back(-1);
    }
  };
  // panels of <= kRtMaxRows rows run on the register-tile engine (build_rt_stream) instead
  const bool rt = PR <= kRtMaxRows;
  for (int64_t p = pb; p < pe && !rt; ++p) {
    const int64_t dc0 = T.dense_ptr[p], dc1 = T.dense_ptr[p + 1];
    if (dc1 == dc0) continue;
    const int64_t q0 = p * PR, nrows = std::min<int64_t>(M, q0 + PR) - q0;
    const int64_t nd = dc1 - dc0, nt = (nd + TW - 1) / TW;
    maxd = std::max(maxd, nd);
    for (int64_t r = 0; r < nrows; ++r) cur[r] = T.drow_ptr[q0 + r];
    const int64_t vt_first = (int64_t)vtiles.size();
    for (int64_t t = 0; t < nt; ++t) {
      const int64_t s_hi = (t + 1) * TW;
      for (int64_t r = 0; r < nrows; ++r) {
        stop[r] = cur[r];
        const int64_t end = T.drow_ptr[q0 + r + 1];
        while (stop[r] < end && T.d_slot[stop[r]] < s_hi) ++stop[r];
      }
      int64_t ra = 0;
      while (ra < std::max<int64_t>(nrows, 1)) {
        int64_t rb = ra, cnt = 0;
        while (rb < nrows && cnt + (stop[rb] - cur[rb]) <= kMaxTileEntries) cnt += stop[rb] - cur[rb], ++rb;
        if (rb == ra) rb = ra + 1;  // cannot happen (a row has <= TW entries per tile)
        pad4();
        VTile v;
        v.ent0 = (int32_t)de.size();
        v.col0 = (int32_t)(dc0 + t * TW);
        v.ncols = (int32_t)(std::min(nd, s_hi) - t * TW);
        int32_t off = 0;
        for (int64_t r = 0; r < TS; ++r) {
          trp.push_back(off);
          if (r >= ra && r < rb && r < nrows) {
            for (int64_t e = cur[r]; e < stop[r]; ++e) {
              int2 x;
              x.x = T.d_slot[e] - (int32_t)(t * TW);
              x.y = *reinterpret_cast<const int32_t*>(&A.val[T.d_cidx[e]]);
              de.push_back(x);
              deo.push_back(d_out[e]);
              ++off;
            }
          }
        }
        pad4();
        v.nent = (int32_t)de.size() - v.ent0;
        vtiles.push_back(v);
        ra = rb;
      }
      for (int64_t r = 0; r < nrows; ++r) cur[r] = stop[r];
    }
    const int64_t nvt = (int64_t)vtiles.size() - vt_first;
    const int64_t nunits = (nvt + kMaxUnitTiles - 1) / kMaxUnitTiles;
    for (int64_t c = 0; c < nunits; ++c) {
      const int64_t t0 = c * kMaxUnitTiles, t1 = std::min(nvt, t0 + kMaxUnitTiles);
      DUnit u{};
      u.q0 = (int32_t)q0;
      u.nrows = (int32_t)nrows;
      u.vt0 = (int32_t)(vt_first + t0);
      u.nvt = (int32_t)(t1 - t0);
      u.split = nunits > 1 ? (int32_t)(n_dslots + c) : -1;
      units.push_back(u);
      if (nunits > 1) dsplit.push_back(make_int2((int)n_dslots, (int)nunits));
    }
    if (nunits > 1) n_dslots += nunits;
  }
  pad4();
  if (rt) SR_TRY(build_rt_stream(h, pb, pe, d_out, P, s));
  P.n_units = (int64_t)units.size();
  P.max_dense_per_panel = maxd;
  P.tile_cols = TW;
  P.trp_stride = TS;
  P.panel_rows = PR;
  P.n_dslots = n_dslots;
  P.dscratch.release();
  P.dscratch_k = 0;
  // persistent phase-D CTAs take units round-robin: largest first balances them; every unit
  // gets a producer blob (DUnit | VTiles), 16-byte aligned
  std::stable_sort(units.begin(), units.end(), [](const DUnit& a, const DUnit& b) { return a.nvt > b.nvt; });
  std::vector<int4> blobs;
  std::vector<int2> blob_meta;
  for (const DUnit& u : units) {
    std::vector<int32_t> rec(8 + 4 * u.nvt, 0);
    std::memcpy(rec.data(), &u, sizeof(DUnit));
    std::memcpy(rec.data() + 8, &vtiles[u.vt0], sizeof(VTile) * u.nvt);
    blob_meta.push_back(make_int2((int)blobs.size(), (int)(rec.size() * 4)));
    for (size_t w = 0; w < rec.size(); w += 4) blobs.push_back(make_int4(rec[w], rec[w + 1], rec[w + 2], rec[w + 3]));
  }
  SR_TRY(P.blobs.upload(blobs, s));
  SR_TRY(P.blob_meta.upload(blob_meta, s));
  SR_TRY(P.units.upload(units, s));
  SR_TRY(P.vtiles.upload(vtiles, s));
  SR_TRY(P.dense_cols.upload(T.dense_cols, s));
  SR_TRY(P.trp.upload(trp, s));
  SR_TRY(P.d_ent.upload(de, s));
  SR_TRY(P.d_oidx.upload(deo, s));
  if (n_dslots > 0) {
    SR_TRY(P.dsplit_info.upload(dsplit, s));
    SR_TRY(P.dsplit_counter.alloc((size_t)n_dslots));
    SR_CUDA_TRY(cudaMemsetAsync(P.dsplit_counter.p, 0, n_dslots * sizeof(int32_t), s));
  }
  {
    std::vector<int32_t> drp((size_t)M + 1);
    for (int64_t q = 0; q <= M; ++q) drp[q] = (int32_t)T.drow_ptr[q];
    SR_TRY(P.drow_ptr.upload(drp, s));
    std::vector<int32_t> pout((size_t)M);
    for (int64_t q = 0; q < M; ++q) pout[q] = sharded ? (int32_t)(q - q0s) : perm1[q];
    SR_TRY(P.pos_xrow.upload(perm1, s));
    SR_TRY(P.pos_out.upload(pout, s));
    std::vector<int32_t> dout((size_t)M);
    for (int64_t q = 0; q < M; ++q) dout[q] = T.drow_ptr[q + 1] > T.drow_ptr[q] ? pout[q] : -1;
    SR_TRY(P.dense_out.upload(dout, s));
  }
  // phase S: remainder rows in perm2 order (restricted to the shard), then zero rows
  std::vector<int2> se;
  std::vector<int32_t> so;
  se.reserve(T.r_col.size());
  so.reserve(T.r_col.size());
  ItemBuilder ib;
  std::vector<int32_t> rows_s;  // the shard's remainder positions in perm2 order
  std::vector<int64_t> soff;    // their offsets in the stream
  int64_t ns = 0;
  for (int32_t q : h->perm2) {
    if (q < q0s || q >= q1s) continue;
    const int64_t len = T.rrow_ptr[q + 1] - T.rrow_ptr[q];
    const bool rmw = T.drow_ptr[q + 1] > T.drow_ptr[q];
    const int32_t out = sharded ? (int32_t)(q - q0s) : perm1[q];
    ib.add_row((int32_t)ns, (int32_t)(ns + len), perm1[q], out, rmw);
    rows_s.push_back(q);
    soff.push_back(ns);
    ns += len;
  }
  se.resize((size_t)ns);
  so.resize((size_t)ns);
#pragma omp parallel for schedule(dynamic, 256)
  for (int64_t i = 0; i < (int64_t)rows_s.size(); ++i) {
    const int32_t q = rows_s[i];
    int64_t o = soff[i];
    for (int64_t e = T.rrow_ptr[q]; e < T.rrow_ptr[q + 1]; ++e, ++o) {
      se[o] = make_int2(T.r_col[e], *reinterpret_cast<const int32_t*>(&A.val[T.r_cidx[e]]));
      so[o] = r_out[e];
    }
  }
  const int64_t n_nonzero = (int64_t)ib.items.size();
  for (int64_t q = q0s; q < q1s; ++q) {
    if (T.drow_ptr[q + 1] == T.drow_ptr[q] && T.rrow_ptr[q + 1] == T.rrow_ptr[q]) {
      const int32_t out = sharded ? (int32_t)(q - q0s) : perm1[q];
      ib.items.push_back(Item{0, 0, perm1[q], out});
      ib.meta.push_back(0u);
    }
  }
  // bytes model
  sr_traffic_model& tm = P.traffic;
  std::memset(&tm, 0, sizeof(tm));
  sparse_traffic(ib, n_nonzero, (int64_t)ib.items.size() - n_nonzero, se, A.N, tm);
  {
    std::vector<uint8_t> seen((size_t)A.N, 0);
    for (const VTile& d : vtiles) {
      tm.dense_col_loads += d.ncols;
      for (int32_t k = d.col0; k < d.col0 + d.ncols; ++k)
        if (!seen[T.dense_cols[k]]) {
          seen[T.dense_cols[k]] = 1;
          ++tm.dense_distinct_cols;
        }
    }
    if (rt) {  // register tiles: every dense column of a panel is gathered once per K pass
      for (int64_t p = pb; p < pe; ++p) {
        for (int64_t k = T.dense_ptr[p]; k < T.dense_ptr[p + 1]; ++k) {
          ++tm.dense_col_loads;
          if (!seen[T.dense_cols[k]]) {
            seen[T.dense_cols[k]] = 1;
            ++tm.dense_distinct_cols;
          }
        }
      }
    }
    tm.dense_panels = P.n_rt + (int64_t)units.size();
    for (int64_t q = q0s; q < q1s; ++q) {
      const bool d = T.drow_ptr[q + 1] > T.drow_ptr[q], r = T.rrow_ptr[q + 1] > T.rrow_ptr[q];
      tm.dense_nnz += T.drow_ptr[q + 1] - T.drow_ptr[q];
      tm.dense_rows += d;
      tm.rmw_rows += d && r;
    }
  }
  se.resize(se.size() + kEntPad, make_int2(0, 0));
  so.resize(so.size() + kEntPad, -1);
  SR_TRY(P.s_ent.upload(se, s));
  SR_TRY(P.s_oidx.upload(so, s));
  SR_TRY(upload_items(P, ib, n_nonzero, s));
  SR_CUDA_TRY(cudaStreamSynchronize(s));
  return SR_OK;
}

int check_params(const sr_reorder_params* p) {
  if (!p) return einval("sr_reorder: params is NULL");
  if (p->siglen <= 0 || p->siglen > 256) return einval("siglen must be in 1..256");
  if (p->bsize <= 0 || p->siglen % p->bsize != 0) return einval("siglen % bsize != 0 (R24)");
  if (p->bsize > 2) {
    set_error("bsize > 2 is not supported by the GPU banding kernel");
    return SR_EUNSUPPORTED;
  }
  if (p->threshold_size < 2) return einval("threshold_size must be >= 2");
  if (p->max_bucket < 0 || p->max_bucket == 1) return einval("max_bucket must be 0 or >= 2");
  if (p->panel_rows < 1 || p->panel_rows > 128) return einval("panel_rows must be in 1..128");
  if (p->dense_min < 1) return einval("dense_min must be >= 1");
  if (p->tile_cols < 1 || p->tile_cols > 1024) return einval("tile_cols must be in 1..1024");
  if (p->mode < 0 || p->mode > 2) return einval("mode must be AUTO, FORCE or OFF");
  if (p->skip_dense_den <= 0 || p->skip_sim_den <= 0 || p->skip_dense_num < 0 || p->skip_sim_num < 0)
    return einval("decision thresholds must be non-negative fractions");
  if (p->world < 1 || p->rank < 0 || p->rank >= p->world) return einval("bad world / rank");
  if (p->auto_dense_min < 0) return einval("auto_dense_min must be >= 0 (0 = dense_min)");
  if (p->reserved0 != 0) return einval("reserved0 must be 0");
  return SR_OK;
}

// LSH + Alg 3 over a column-sorted CSR (rows = the matrix being reordered).
int reorder_round(const int64_t* rowptr, const int32_t* col, int64_t M, const sr_reorder_params& p,
                  cudaStream_t s, std::vector<int32_t>& perm, int64_t* E, double* t_lsh, double* t_cl) {
  HostVec<uint64_t> pairs, by_key;
  HostVec<uint32_t> inter, uni;
  const double t0 = now_s();
  SR_TRY(lsh_candidates(rowptr, col, M, rowptr[M], p, s, pairs, inter, uni, E, &by_key));
  const double t1 = now_s();
  perm.resize((size_t)M);
  cluster_rows(M, rowptr, col, (int64_t)pairs.size(), pairs.data(), inter.data(), uni.data(),
               p.threshold_size, perm.data(), by_key.empty() ? nullptr : by_key.data());
  *t_lsh += t1 - t0;
  *t_cl += now_s() - t1;
  return SR_OK;
}

// Restores a handle's plan state (parameters, orders, tiling, stats) unless committed: a failed
// sr_reorder / sr_plan_load leaves the handle as it was (its identity plan stays usable).
struct PlanRollback {
  sr_csr_s* h;
  bool armed = true;
  sr_reorder_params params;
  std::vector<int32_t> perm1, perm2;
  Tiling tiles;
  sr_plan_stats stats;
  explicit PlanRollback(sr_csr_s* h_)
      : h(h_), params(h_->params), perm1(h_->perm1), perm2(h_->perm2), tiles(h_->tiles), stats(h_->stats) {}
  ~PlanRollback() {
    if (!armed) return;
    h->params = params;
    h->perm1 = std::move(perm1);
    h->perm2 = std::move(perm2);
    h->tiles = std::move(tiles);
    h->stats = stats;
  }
  void commit() { armed = false; }
};

// Shard selection + device execution plan of the plan held in h (perm1, its tiling, perm2).
int finish_plan(sr_csr_s* h, cudaStream_t s) {
  const sr_reorder_params* p = &h->params;
  const Tiling& T = h->tiles;
  const int64_t M = h->A.M;
  sr_plan_stats& st = h->stats;
  // shard: contiguous nnz-balanced panel ranges
  int64_t pb = 0, pe = T.npanels;
  if (p->world > 1) {
    std::vector<int64_t> w((size_t)T.npanels), cuts((size_t)p->world + 1);
    for (int64_t q = 0; q < T.npanels; ++q) {
      const int64_t a = q * p->panel_rows, b = std::min<int64_t>(M, a + p->panel_rows);
      w[q] = (T.drow_ptr[b] - T.drow_ptr[a]) + (T.rrow_ptr[b] - T.rrow_ptr[a]);
    }
    partition_panels(T.npanels, w.data(), p->world, cuts.data());
    pb = cuts[p->rank];
    pe = cuts[p->rank + 1];
  }
  st.shard_panel_begin = pb;
  st.shard_panel_end = pe;
  const double t0 = now_s();
  SR_TRY(build_exec_plan(h, pb, pe, s));
  st.t_plan_s = now_s() - t0;
  st.shard_nrows = (int64_t)h->shard_rows.size();
  st.shard_nnz = (int64_t)h->shard_nnz_ids.size();
  h->reordered = true;
  return SR_OK;
}

}  // namespace
}  // namespace sr

using namespace sr;

extern "C" {

const char* sr_last_error(void) { return g_err.c_str(); }
const char* sr_version(void) { return "sr 0.1 (sm_100a)"; }

void sr_default_params(sr_reorder_params* p) {
  if (!p) return;
  std::memset(p, 0, sizeof(*p));
  p->siglen = 128;
  p->bsize = 2;
  p->threshold_size = 256;
  p->max_bucket = 32;
  p->seed = 4;
  p->panel_rows = 64;
  p->dense_min = 2;
  p->tile_cols = 64;
  p->mode = SR_REORDER_AUTO;
  p->skip_dense_num = 1;
  p->skip_dense_den = 10;
  p->skip_sim_num = 1;
  p->skip_sim_den = 10;
  p->world = 1;
  p->rank = 0;
}

int sr_csr_create(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t* rowptr,
                  const int32_t* colidx, const float* vals, int device, sr_csr* out) {
  if (!out) return einval("sr_csr_create: out is NULL");
  *out = nullptr;
  if (nrows < 0 || ncols < 0 || nnz < 0) return einval("negative size");
  if (nrows >= (1ll << 31) || ncols >= (1ll << 31) || nnz >= (1ll << 31)) {
    set_error("nrows, ncols and nnz must be < 2^31");
    return SR_EUNSUPPORTED;
  }
  if (!rowptr || (nnz > 0 && (!colidx || !vals))) return einval("NULL CSR array");
  if (rowptr[0] != 0 || rowptr[nrows] != nnz) return einval("rowptr[0] != 0 or rowptr[M] != nnz");
  for (int64_t i = 0; i < nrows; ++i)
    if (rowptr[i + 1] < rowptr[i]) return einval("rowptr is decreasing at row " + std::to_string(i));
  auto* h = new (std::nothrow) sr_csr_s();
  if (!h) {
    set_error("out of host memory");
    return SR_ENOMEM;
  }
  h->device = device;
  HostCSR& A = h->A;
  A.M = nrows;
  A.N = ncols;
  A.rowptr.assign(rowptr, rowptr + nrows + 1);
  A.col.resize((size_t)nnz);
  A.val.resize((size_t)nnz);
  bool bad = false, unsorted = false;
#pragma omp parallel for schedule(dynamic, 1024) reduction(|| : bad, unsorted)
  for (int64_t i = 0; i < nrows; ++i) {
    for (int64_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
      if (colidx[e] < 0 || colidx[e] >= ncols) bad = true;
      if (e > rowptr[i] && colidx[e] <= colidx[e - 1]) unsorted = true;
    }
  }
  if (bad) {
    delete h;
    return einval("column index out of range");
  }
  if (!unsorted) {
    std::memcpy(A.col.data(), colidx, nnz * sizeof(int32_t));
    std::memcpy(A.val.data(), vals, nnz * sizeof(float));
    A.identity_pos = true;
  } else {
    A.identity_pos = false;
    A.opos.resize((size_t)nnz);
    bool dup = false;
#pragma omp parallel for schedule(dynamic, 1024) reduction(|| : dup)
    for (int64_t i = 0; i < nrows; ++i) {
      const int64_t b = rowptr[i], e = rowptr[i + 1];
      std::vector<int64_t> idx((size_t)(e - b));
      std::iota(idx.begin(), idx.end(), b);
      std::sort(idx.begin(), idx.end(), [&](int64_t x, int64_t y) {
        return colidx[x] != colidx[y] ? colidx[x] < colidx[y] : x < y;
      });
      for (int64_t t = 0; t < e - b; ++t) {
        A.col[b + t] = colidx[idx[t]];
        A.val[b + t] = vals[idx[t]];
        A.opos[b + t] = (int32_t)idx[t];
        if (t > 0 && A.col[b + t] == A.col[b + t - 1]) dup = true;
      }
    }
    if (dup) {
      delete h;
      return einval("duplicate (row, col) entry");
    }
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    cudaGetLastError();
    delete h;
    set_error("sr_csr_create: no such CUDA device " + std::to_string(device));
    return SR_ECUDA;
  }
  DeviceGuard dg(device);
  if (cudaStreamCreateWithFlags(&h->init_stream, cudaStreamNonBlocking) != cudaSuccess) {
    cudaGetLastError();
    delete h;
    set_error("cudaStreamCreate failed");
    return SR_ECUDA;
  }
  // the identity plan (P:101 row-wise kernels) is built on first use (ensure_plan), so a handle
  // that is reordered or given a saved plan right away never uploads it
  sr_default_params(&h->params);
  h->perm1.resize((size_t)nrows);
  std::iota(h->perm1.begin(), h->perm1.end(), 0);
  h->stats.nnz = nnz;
  *out = h;
  return SR_OK;
}

int sr_reorder(sr_csr h, const sr_reorder_params* p, sr_stream stream) {
  if (!h) return einval("sr_reorder: NULL handle");
  SR_TRY(check_params(p));
  if (h->reordered) {
    set_error("sr_reorder: the handle already has a plan");
    return SR_ESTATE;
  }
  DeviceGuard dg(h->device);
  cudaStream_t s = stream ? (cudaStream_t)stream : h->init_stream;
  const double t_start = now_s();
  PlanRollback rollback(h);
  h->params = *p;
  const HostCSR& A = h->A;
  const int64_t M = A.M, nnz = A.nnz();
  sr_plan_stats& st = h->stats;
  std::memset(&st, 0, sizeof(st));
  st.nnz = nnz;
  std::vector<int32_t> ident((size_t)M);
  std::iota(ident.begin(), ident.end(), 0);
  // DenseRatio of the original order under the decision's dense criterion (R28)
  double t0 = now_s();
  const int32_t dense_min0 = p->auto_dense_min > 0 ? p->auto_dense_min : p->dense_min;
  Tiling t_id;
  const bool tile_ident = p->mode == SR_REORDER_OFF;  // OFF plans are the identity tiling itself
  if (tile_ident) {
    tile_rows(A, ident, p->panel_rows, dense_min0, t_id);
    st.dense0 = t_id.n_dense();
  } else {  // only the count decides round 1 (the tiles are built below if it is skipped)
    st.dense0 = dense_count(A, ident, p->panel_rows, dense_min0);
  }
  st.t_tile_s += now_s() - t0;
  bool round1 = p->mode == SR_REORDER_FORCE;
  if (p->mode == SR_REORDER_AUTO)
    round1 = !((unsigned __int128)st.dense0 * (uint64_t)p->skip_dense_den >
               (unsigned __int128)p->skip_dense_num * (uint64_t)nnz);
  if (round1) {
    SR_TRY(reorder_round(A.rowptr.data(), A.col.data(), M, *p, s, h->perm1, &st.E1, &st.t_lsh1_s,
                         &st.t_cluster1_s));
    t0 = now_s();
    tile_rows(A, h->perm1, p->panel_rows, p->dense_min, h->tiles);
    st.t_tile_s += now_s() - t0;
  } else {
    h->perm1 = ident;
    if (!tile_ident || dense_min0 != p->dense_min) {  // the plan tiles with the execution threshold
      t0 = now_s();
      tile_rows(A, ident, p->panel_rows, p->dense_min, t_id);
      st.t_tile_s += now_s() - t0;
    }
    h->tiles = std::move(t_id);
  }
  st.round1 = round1 ? 1 : 0;
  const Tiling& T = h->tiles;
  st.dense1 = T.n_dense();
  st.npanels = T.npanels;
  st.ndense_cols = (int64_t)T.dense_cols.size();
  for (int64_t q = 0; q < T.npanels; ++q)
    st.ntiles += (T.dense_ptr[q + 1] - T.dense_ptr[q] + p->tile_cols - 1) / p->tile_cols;
  avgsim_positions(T, &st.avgsim_num, &st.avgsim_den);
  bool round2 = p->mode == SR_REORDER_FORCE;
  if (p->mode == SR_REORDER_AUTO)
    round2 = !((unsigned __int128)st.avgsim_num * (uint64_t)p->skip_sim_den >
               (unsigned __int128)p->skip_sim_num * st.avgsim_den);
  st.round2 = round2 ? 1 : 0;
  std::vector<int32_t> order;
  if (round2) {
    SR_TRY(reorder_round(T.rrow_ptr.data(), T.r_col.data(), M, *p, s, order, &st.E2, &st.t_lsh2_s,
                         &st.t_cluster2_s));
  } else {
    order = ident;
  }
  h->perm2.clear();
  for (int32_t q : order)
    if (T.rrow_ptr[q + 1] > T.rrow_ptr[q]) h->perm2.push_back(q);
  st.n_perm2 = (int64_t)h->perm2.size();
  const double t_fin = now_s();
  SR_TRY(finish_plan(h, s));
  const double t_trim = now_s();
  cudaStreamSynchronize(s);
  if (!getenv("SR_POOL_KEEP")) trim_pool(h->device);  // give back the LSH rounds' pooled temporaries
  st.t_total_s = now_s() - t_start;
  if (getenv("SR_DEBUG_REORDER"))
    fprintf(stderr, "sr_reorder: total %.3f s = lsh %.3f + %.3f, cluster %.3f + %.3f, tile %.3f, finish_plan %.3f "
            "(exec plan %.3f), trim %.3f, other %.3f\n", st.t_total_s, st.t_lsh1_s, st.t_lsh2_s, st.t_cluster1_s,
            st.t_cluster2_s, st.t_tile_s, t_trim - t_fin, st.t_plan_s, now_s() - t_trim,
            st.t_total_s - (st.t_lsh1_s + st.t_lsh2_s + st.t_cluster1_s + st.t_cluster2_s + st.t_tile_s +
                            (now_s() - t_fin)));
  rollback.commit();
  return SR_OK;
}

int sr_spmm(sr_csr h, const float* B, int64_t K, int64_t ldb, float* C, int64_t ldc, sr_stream stream) {
  if (!h) return einval("sr_spmm: NULL handle");
  if (K < 1 || ldb < K || ldc < K) return einval("sr_spmm: need K >= 1, ldb >= K, ldc >= K");
  const int64_t rows_out = h->params.world > 1 && h->reordered ? (int64_t)h->shard_rows.size() : h->A.M;
  if ((rows_out > 0 && !C) || (h->A.nnz() > 0 && !B)) return einval("sr_spmm: NULL operand");
  if (rows_out == 0) return SR_OK;
  DeviceGuard dg(h->device);
  SR_TRY(ensure_plan(h));
  return launch_spmm(h, B, K, ldb, C, ldc, (cudaStream_t)stream, &h->last_launches);
}

int sr_sddmm(sr_csr h, const float* X, int64_t ldx, const float* Y, int64_t ldy, int64_t K, float* out,
             sr_stream stream) {
  if (!h) return einval("sr_sddmm: NULL handle");
  if (K < 1 || ldx < K || ldy < K) return einval("sr_sddmm: need K >= 1, ldx >= K, ldy >= K");
  if (h->A.nnz() == 0) return SR_OK;
  if (!X || !Y || !out) return einval("sr_sddmm: NULL operand");
  DeviceGuard dg(h->device);
  SR_TRY(ensure_plan(h));
  return launch_sddmm(h, X, ldx, Y, ldy, K, out, (cudaStream_t)stream, &h->last_launches);
}

int sr_destroy(sr_csr h) {
  if (!h) return SR_OK;
  {
    DeviceGuard dg(h->device);
    cudaDeviceSynchronize();
    if (h->init_stream) cudaStreamDestroy(h->init_stream);
    for (cudaEvent_t e : h->plan.ev)
      if (e) cudaEventDestroy(e);
    delete h;
  }
  return SR_OK;
}

int sr_get_perm(sr_csr h, int which, int32_t* out, int64_t cap, int64_t* len) {
  if (!h || !len) return einval("sr_get_perm: NULL argument");
  const std::vector<int32_t>* v = which == 1 ? &h->perm1 : which == 2 ? &h->perm2 : nullptr;
  if (!v) return einval("sr_get_perm: which must be 1 or 2");
  *len = (int64_t)v->size();
  if (cap < *len) return out ? einval("sr_get_perm: capacity too small") : SR_OK;
  if (out && !v->empty()) std::memcpy(out, v->data(), v->size() * sizeof(int32_t));
  return SR_OK;
}

int sr_get_params(sr_csr h, sr_reorder_params* out) {
  if (!h || !out) return einval("sr_get_params: NULL argument");
  *out = h->params;
  return SR_OK;
}

int sr_get_plan_stats(sr_csr h, sr_plan_stats* out) {
  if (!h || !out) return einval("sr_get_plan_stats: NULL argument");
  *out = h->stats;
  return SR_OK;
}

int sr_export_tiles(sr_csr h, int64_t* dense_ptr, int32_t* dense_cols, int64_t* drow_ptr, int32_t* d_slot,
                    int64_t* d_pos, int64_t* rrow_ptr, int32_t* r_col, int64_t* r_pos) {
  if (!h) return einval("sr_export_tiles: NULL handle");
  if (!h->reordered) {
    set_error("sr_export_tiles: no plan yet (call sr_reorder)");
    return SR_ESTATE;
  }
  const Tiling& T = h->tiles;
  const HostCSR& A = h->A;
  auto orig = [&](int64_t c) -> int64_t { return A.identity_pos ? c : A.opos[c]; };
  if (dense_ptr) std::copy(T.dense_ptr.begin(), T.dense_ptr.end(), dense_ptr);
  if (dense_cols) std::copy(T.dense_cols.begin(), T.dense_cols.end(), dense_cols);
  if (drow_ptr) std::copy(T.drow_ptr.begin(), T.drow_ptr.end(), drow_ptr);
  if (d_slot) std::copy(T.d_slot.begin(), T.d_slot.end(), d_slot);
  if (d_pos)
    for (size_t e = 0; e < T.d_cidx.size(); ++e) d_pos[e] = orig(T.d_cidx[e]);
  if (rrow_ptr) std::copy(T.rrow_ptr.begin(), T.rrow_ptr.end(), rrow_ptr);
  if (r_col) std::copy(T.r_col.begin(), T.r_col.end(), r_col);
  if (r_pos)
    for (size_t e = 0; e < T.r_cidx.size(); ++e) r_pos[e] = orig(T.r_cidx[e]);
  return SR_OK;
}

int sr_shard_rows(sr_csr h, int32_t* rows_out, int64_t cap, int64_t* len) {
  if (!h || !len) return einval("sr_shard_rows: NULL argument");
  std::vector<int32_t> all;
  const std::vector<int32_t>* v = &h->shard_rows;
  if (!h->reordered) {
    all = h->perm1;
    v = &all;
  }
  *len = (int64_t)v->size();
  if (cap < *len) return rows_out ? einval("sr_shard_rows: capacity too small") : SR_OK;
  if (rows_out && !v->empty()) std::memcpy(rows_out, v->data(), v->size() * sizeof(int32_t));
  return SR_OK;
}

int sr_shard_nnz_ids(sr_csr h, int64_t* ids_out, int64_t cap, int64_t* len) {
  if (!h || !len) return einval("sr_shard_nnz_ids: NULL argument");
  if (!h->reordered) {
    set_error("sr_shard_nnz_ids: no plan yet");
    return SR_ESTATE;
  }
  *len = (int64_t)h->shard_nnz_ids.size();
  if (cap < *len) return ids_out ? einval("sr_shard_nnz_ids: capacity too small") : SR_OK;
  if (ids_out && *len) std::memcpy(ids_out, h->shard_nnz_ids.data(), *len * sizeof(int64_t));
  return SR_OK;
}

int sr_get_traffic_model(sr_csr h, sr_traffic_model* out) {
  if (!h || !out) return einval("sr_get_traffic_model: NULL argument");
  *out = h->plan.traffic;
  return SR_OK;
}

int sr_set_profiling(sr_csr h, int enable) {
  if (!h) return einval("sr_set_profiling: NULL handle");
  h->plan.profiling = enable != 0;
  return SR_OK;
}

int sr_last_kernel_times(sr_csr h, int32_t* kinds, float* ms, int32_t cap, int32_t* n) {
  if (!h || !n) return einval("sr_last_kernel_times: NULL argument");
  DevPlan& P = h->plan;
  *n = P.nrec;
  if (cap < P.nrec) return (kinds || ms) ? einval("sr_last_kernel_times: capacity too small") : SR_OK;
  DeviceGuard dg(h->device);
  for (int32_t i = 0; i < P.nrec; ++i) {
    SR_CUDA_TRY(cudaEventSynchronize(P.ev[2 * i + 1]));
    float t = 0.f;
    SR_CUDA_TRY(cudaEventElapsedTime(&t, P.ev[2 * i], P.ev[2 * i + 1]));
    if (kinds) kinds[i] = P.kinds[i];
    if (ms) ms[i] = t;
  }
  return SR_OK;
}

int sr_last_launch_count(sr_csr h, int32_t* n) {
  if (!h || !n) return einval("sr_last_launch_count: NULL argument");
  *n = h->last_launches;
  return SR_OK;
}

int sr_host_cluster(int64_t M, const int64_t* rowptr, const int32_t* colidx, int64_t npairs,
                    const uint64_t* pairs, const uint32_t* inter, const uint32_t* uni, int32_t threshold_size,
                    int32_t* perm) {
  if (M < 0 || !rowptr || !perm || (npairs > 0 && !pairs) || threshold_size < 1)
    return einval("sr_host_cluster: bad argument");
  for (int64_t e = 0; e < npairs; ++e) {
    const uint64_t i = pairs[e] >> 32, j = pairs[e] & 0xFFFFFFFFu;
    if (i >= j || (int64_t)j >= M || (e > 0 && pairs[e] <= pairs[e - 1]))
      return einval("sr_host_cluster: pairs must be sorted, unique, i < j < M");
  }
  cluster_rows(M, rowptr, colidx, npairs, pairs, inter, uni, threshold_size, perm, pairs);  // key-sorted (checked)
  return SR_OK;
}

int sr_scatter_rows(const float* src, int64_t lds, const int32_t* rows, int64_t n, int64_t K, float* dst,
                    int64_t ldd, sr_stream stream) {
  if (n < 0 || K < 1 || lds < K || ldd < K || (n > 0 && (!src || !rows || !dst)))
    return einval("sr_scatter_rows: bad argument");
  return launch_scatter_rows(src, lds, rows, n, K, dst, ldd, (cudaStream_t)stream);
}

int sr_scatter_values(const float* src, const int64_t* ids, int64_t n, float* dst, sr_stream stream) {
  if (n < 0 || (n > 0 && (!src || !ids || !dst))) return einval("sr_scatter_values: bad argument");
  return launch_scatter_values(src, ids, n, dst, (cudaStream_t)stream);
}

int sr_host_partition(int64_t npanels, const int64_t* weights, int32_t G, int64_t* cuts) {
  if (npanels < 0 || G < 1 || !cuts || (npanels > 0 && !weights)) return einval("sr_host_partition: bad argument");
  partition_panels(npanels, weights, G, cuts);
  return SR_OK;
}

}  // extern "C"

// ------------------------------------------------------------------ offline plans
namespace sr {
namespace {
constexpr char kPlanMagic[8] = {'S', 'R', 'P', 'L', 'A', 'N', '0', '1'};
constexpr uint32_t kPlanVersion = 2;  // 2: sr_reorder_params gained auto_dense_min

// 64-bit hash of a byte range (word-wise multiply-xorshift; not cryptographic).
uint64_t hash_bytes(const void* p, size_t n, uint64_t h) {
  const unsigned char* b = static_cast<const unsigned char*>(p);
  size_t i = 0;
  for (; i + 8 <= n; i += 8) {
    uint64_t w;
    std::memcpy(&w, b + i, 8);
    h ^= w * 0x9E3779B97F4A7C15ull;
    h = (h << 27 | h >> 37) * 0xBF58476D1CE4E5B9ull;
  }
  for (; i < n; ++i) h = (h ^ b[i]) * 0x100000001B3ull;
  return h ^ (h >> 31);
}

uint64_t matrix_fingerprint(const HostCSR& A) {
  uint64_t h = hash_bytes(&A.M, 8, 0x5252504C414E3031ull);
  h = hash_bytes(&A.N, 8, h);
  h = hash_bytes(A.rowptr.data(), A.rowptr.size() * 8, h);
  return hash_bytes(A.col.data(), A.col.size() * 4, h);
}

struct PlanWriter {
  std::vector<unsigned char> b;
  template <typename T>
  void put(const T& v) { put_raw(&v, sizeof(T)); }
  void put_raw(const void* p, size_t n) {
    const unsigned char* c = static_cast<const unsigned char*>(p);
    b.insert(b.end(), c, c + n);
  }
};

struct PlanReader {
  const unsigned char* p;
  size_t n, off = 0;
  bool ok = true;
  bool get_raw(void* dst, size_t k) {
    if (!ok || off + k > n) return ok = false;
    std::memcpy(dst, p + off, k);
    off += k;
    return true;
  }
  template <typename T>
  bool get(T& v) { return get_raw(&v, sizeof(T)); }
};
}  // namespace
}  // namespace sr

extern "C" {

int sr_plan_save(sr_csr h, void* buf, int64_t cap, int64_t* len) {
  if (!h || !len) return einval("sr_plan_save: NULL argument");
  if (!h->reordered) {
    set_error("sr_plan_save: the handle has no plan (call sr_reorder or sr_plan_load first)");
    return SR_ESTATE;
  }
  PlanWriter w;
  w.put_raw(kPlanMagic, 8);
  w.put(kPlanVersion);
  w.put((uint32_t)0);
  w.put(h->A.M);
  w.put(h->A.N);
  const int64_t nnz = h->A.nnz();
  w.put(nnz);
  w.put(matrix_fingerprint(h->A));
  sr_reorder_params p = h->params;
  p.world = 1;
  p.rank = 0;
  w.put(p);
  sr_plan_stats st = h->stats;  // shard fields describe the whole matrix in the image
  st.shard_panel_begin = 0;
  st.shard_panel_end = st.npanels;
  st.shard_nrows = h->A.M;
  st.shard_nnz = nnz;
  st.t_lsh1_s = st.t_cluster1_s = st.t_tile_s = st.t_lsh2_s = st.t_cluster2_s = st.t_total_s = st.t_plan_s = 0.0;
  w.put(st);
  w.put((int64_t)h->perm1.size());
  w.put_raw(h->perm1.data(), h->perm1.size() * 4);
  w.put((int64_t)h->perm2.size());
  w.put_raw(h->perm2.data(), h->perm2.size() * 4);
  w.put(hash_bytes(w.b.data(), w.b.size(), 0));
  *len = (int64_t)w.b.size();
  if (!buf) return SR_OK;
  if (cap < *len) return einval("sr_plan_save: capacity too small");
  std::memcpy(buf, w.b.data(), w.b.size());
  return SR_OK;
}

int sr_plan_load(sr_csr h, const void* buf, int64_t len, int32_t world, int32_t rank, sr_stream stream) {
  if (!h || !buf || len <= 0) return einval("sr_plan_load: NULL argument");
  if (h->reordered) {
    set_error("sr_plan_load: the handle already has a plan");
    return SR_ESTATE;
  }
  const double t_start = now_s();
  PlanReader r{static_cast<const unsigned char*>(buf), (size_t)len};
  if (len < 8 + 8 || std::memcmp(buf, kPlanMagic, 8) != 0) return einval("sr_plan_load: not a plan image");
  uint64_t sum = 0;
  std::memcpy(&sum, r.p + len - 8, 8);
  if (hash_bytes(buf, (size_t)len - 8, 0) != sum) return einval("sr_plan_load: checksum mismatch (corrupted image)");
  char magic[8];
  uint32_t ver = 0, res = 0;
  int64_t M = 0, N = 0, nnz = 0, len1 = 0, len2 = 0;
  uint64_t fp = 0;
  sr_reorder_params p;
  sr_plan_stats st;
  r.get_raw(magic, 8);
  r.get(ver);
  r.get(res);
  r.get(M);
  r.get(N);
  r.get(nnz);
  r.get(fp);
  r.get(p);
  r.get(st);
  if (!r.ok || ver != kPlanVersion) return einval("sr_plan_load: unsupported image version");
  const HostCSR& A = h->A;
  if (M != A.M || N != A.N || nnz != A.nnz() || fp != matrix_fingerprint(A))
    return einval("sr_plan_load: the image belongs to another matrix");
  p.world = world;
  p.rank = rank;
  SR_TRY(check_params(&p));
  if (!r.get(len1) || len1 != M) return einval("sr_plan_load: bad perm1 length");
  std::vector<int32_t> perm1((size_t)M), perm2;
  if (!r.get_raw(perm1.data(), (size_t)M * 4) || !r.get(len2) || len2 < 0 || len2 > M)
    return einval("sr_plan_load: truncated image");
  perm2.resize((size_t)len2);
  if (!r.get_raw(perm2.data(), (size_t)len2 * 4) || r.off + 8 != (size_t)len)
    return einval("sr_plan_load: truncated image");
  {  // perm1 must be a permutation of [0, M)
    std::vector<uint8_t> seen((size_t)M, 0);
    for (int32_t v : perm1) {
      if (v < 0 || v >= M || seen[v]) return einval("sr_plan_load: perm1 is not a permutation");
      seen[v] = 1;
    }
  }
  DeviceGuard dg(h->device);
  cudaStream_t s = stream ? (cudaStream_t)stream : h->init_stream;
  PlanRollback rollback(h);
  h->params = p;
  const double t0 = now_s();
  Tiling T;
  tile_rows(A, perm1, p.panel_rows, p.dense_min, T);
  {  // perm2 must list every non-empty remainder position exactly once
    std::vector<uint8_t> seen((size_t)M, 0);
    int64_t nonempty = 0;
    for (int64_t q = 0; q < M; ++q) nonempty += T.rrow_ptr[q + 1] > T.rrow_ptr[q];
    for (int32_t q : perm2) {
      if (q < 0 || q >= M || seen[q] || T.rrow_ptr[q + 1] == T.rrow_ptr[q])
        return einval("sr_plan_load: perm2 does not match the tiling of perm1");
      seen[q] = 1;
    }
    if (nonempty != len2) return einval("sr_plan_load: perm2 does not match the tiling of perm1");
  }
  h->perm1 = std::move(perm1);
  h->perm2 = std::move(perm2);
  h->tiles = std::move(T);
  st.t_lsh1_s = st.t_cluster1_s = st.t_lsh2_s = st.t_cluster2_s = 0.0;
  st.t_tile_s = now_s() - t0;
  h->stats = st;
  SR_TRY(finish_plan(h, s));
  h->stats.t_total_s = now_s() - t_start;
  rollback.commit();
  return SR_OK;
}

int sr_trial(const sr_csr* cands, int32_t n, int32_t op, const float* U, int64_t ldu, const float* V, int64_t ldv,
             int64_t K, float* out, int64_t ldo, int32_t reps, sr_stream stream, int32_t* best, float* ms) {
  if (!cands || n < 1 || !best || reps < 1) return einval("sr_trial: bad argument");
  if (op != SR_OP_SPMM && op != SR_OP_SDDMM) return einval("sr_trial: op must be SR_OP_SPMM or SR_OP_SDDMM");
  for (int32_t i = 0; i < n; ++i) {
    if (!cands[i]) return einval("sr_trial: NULL candidate");
    const sr_csr_s* a = cands[0];
    const sr_csr_s* b = cands[i];
    const bool sa = a->reordered && a->params.world > 1, sb = b->reordered && b->params.world > 1;
    if (a->A.M != b->A.M || a->A.N != b->A.N || a->A.nnz() != b->A.nnz() || sa || sb || a->device != b->device)
      return einval("sr_trial: candidates must be single-GPU plans of one matrix on one device");
  }
  DeviceGuard dg(cands[0]->device);
  cudaStream_t s = (cudaStream_t)stream;
  cudaEvent_t e0, e1;
  SR_CUDA_TRY(cudaEventCreate(&e0));
  if (cudaEventCreate(&e1) != cudaSuccess) {
    cudaEventDestroy(e0);
    cudaGetLastError();
    set_error("sr_trial: cudaEventCreate failed");
    return SR_ECUDA;
  }
  int rc = SR_OK;
  float best_ms = 0.f;
  *best = 0;
  for (int32_t i = 0; i < n && rc == SR_OK; ++i) {
    auto call = [&]() {
      return op == SR_OP_SPMM ? sr_spmm(cands[i], U, K, ldu, out, ldo, stream)
                              : sr_sddmm(cands[i], U, ldu, V, ldv, K, out, stream);
    };
    if ((rc = call()) != SR_OK) break;  // warm-up
    std::vector<float> t((size_t)reps);
    for (int32_t k = 0; k < reps && rc == SR_OK; ++k) {
      cudaEventRecord(e0, s);
      if ((rc = call()) != SR_OK) break;
      cudaEventRecord(e1, s);
      if (cudaEventSynchronize(e1) != cudaSuccess || cudaEventElapsedTime(&t[k], e0, e1) != cudaSuccess) {
        cudaGetLastError();
        set_error("sr_trial: timing failed");
        rc = SR_ECUDA;
      }
    }
    if (rc != SR_OK) break;
    std::sort(t.begin(), t.end());
    const float med = t[(size_t)reps / 2];
    if (ms) ms[i] = med;
    if (i == 0 || med < best_ms) {
      best_ms = med;
      *best = i;
    }
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return rc;
}

}  // extern "C"

extern "C" int sr_set_values(sr_csr h, const float* vals, sr_stream stream) {
  if (!h) return einval("sr_set_values: NULL handle");
  const int64_t n = h->reordered ? (int64_t)h->shard_nnz_ids.size() : h->A.nnz();
  if (n == 0) return SR_OK;
  if (!vals) return einval("sr_set_values: NULL values");
  DeviceGuard dg(h->device);
  SR_TRY(ensure_plan(h));
  DevPlan& P = h->plan;
  cudaStream_t s = (cudaStream_t)stream;
  SR_TRY(launch_set_values(P.s_ent.p, P.s_oidx.p, (int64_t)P.s_ent.n, vals, s));
  if (P.n_units > 0) SR_TRY(launch_set_values(P.d_ent.p, P.d_oidx.p, (int64_t)P.d_ent.n, vals, s));
  if (P.n_rt > 0) SR_TRY(launch_set_values(P.rt_ent.p, P.rt_oidx.p, (int64_t)P.rt_ent.n, vals, s));
  return SR_OK;
}
