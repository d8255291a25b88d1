// ASpT row-panel tiler (Fig 3; Fig 4) and the AvgSim indicator
// (P:259-265).  Host C++/OpenMP: panels are independent, so they are tiled in parallel
// into per-panel buffers and concatenated.
//   panel p = positions [p·P, min((p+1)·P, M)) of the row order perm;
//   cnt[c]  = rows of the panel containing c;  D_p = {c : cnt[c] >= dense_min} ordered by
//             (cnt desc, c asc) (R18);  slot = index in D_p;  everything else is remainder.
#include <algorithm>
#include <cstring>
#include <vector>

#ifdef _OPENMP
#include <omp.h>
#endif

#include "internal.h"

namespace sr {

namespace {
struct PanelOut {
  std::vector<int32_t> dcols;
  std::vector<int32_t> dcount;  // per row of the panel
  std::vector<int32_t> rcount;
  std::vector<int32_t> d_slot;
  std::vector<int64_t> d_cidx;
  std::vector<int32_t> r_col;
  std::vector<int64_t> r_cidx;
};
}  // namespace

void tile_rows(const HostCSR& A, const std::vector<int32_t>& perm, int32_t P, int32_t dense_min,
               Tiling& t) {
  const int64_t M = A.M, N = A.N;
  const int64_t npanels = (M + P - 1) / P;
  std::vector<PanelOut> out((size_t)npanels);
#pragma omp parallel
  {
    std::vector<int32_t> cnt((size_t)N, 0), slot((size_t)N, -1);
    std::vector<int32_t> touched;
    std::vector<std::pair<int32_t, int64_t>> row_d;
#pragma omp for schedule(dynamic, 4)
    for (int64_t p = 0; p < npanels; ++p) {
      PanelOut& o = out[(size_t)p];
      const int64_t q0 = p * P, q1 = std::min<int64_t>(M, q0 + P);
      touched.clear();
      for (int64_t q = q0; q < q1; ++q) {
        const int64_t r = perm[q];
        for (int64_t e = A.rowptr[r]; e < A.rowptr[r + 1]; ++e) {
          const int32_t c = A.col[e];
          if (cnt[c]++ == 0) touched.push_back(c);
        }
      }
      for (int32_t c : touched)
        if (cnt[c] >= dense_min) o.dcols.push_back(c);
      std::sort(o.dcols.begin(), o.dcols.end(), [&](int32_t x, int32_t y) {
        return cnt[x] != cnt[y] ? cnt[x] > cnt[y] : x < y;
      });
      for (size_t s = 0; s < o.dcols.size(); ++s) slot[o.dcols[s]] = (int32_t)s;
      o.dcount.resize(q1 - q0);
      o.rcount.resize(q1 - q0);
      for (int64_t q = q0; q < q1; ++q) {
        const int64_t r = perm[q];
        row_d.clear();
        int32_t nr = 0;
        for (int64_t e = A.rowptr[r]; e < A.rowptr[r + 1]; ++e) {
          const int32_t c = A.col[e];
          if (slot[c] >= 0) {
            row_d.emplace_back(slot[c], e);
          } else {
            o.r_col.push_back(c);
            o.r_cidx.push_back(e);
            ++nr;
          }
        }
        std::sort(row_d.begin(), row_d.end());
        for (auto& se : row_d) {
          o.d_slot.push_back(se.first);
          o.d_cidx.push_back(se.second);
        }
        o.dcount[q - q0] = (int32_t)row_d.size();
        o.rcount[q - q0] = nr;
      }
      for (int32_t c : touched) {
        cnt[c] = 0;
        slot[c] = -1;
      }
    }
  }
  // concatenate
  t.npanels = npanels;
  t.dense_ptr.assign((size_t)npanels + 1, 0);
  t.drow_ptr.assign((size_t)M + 1, 0);
  t.rrow_ptr.assign((size_t)M + 1, 0);
  std::vector<int64_t> doff((size_t)npanels + 1, 0), roff((size_t)npanels + 1, 0);
  for (int64_t p = 0; p < npanels; ++p) {
    t.dense_ptr[p + 1] = t.dense_ptr[p] + (int64_t)out[p].dcols.size();
    doff[p + 1] = doff[p] + (int64_t)out[p].d_slot.size();
    roff[p + 1] = roff[p] + (int64_t)out[p].r_col.size();
  }
  t.dense_cols.resize((size_t)t.dense_ptr[npanels]);
  t.d_slot.resize((size_t)doff[npanels]);
  t.d_cidx.resize((size_t)doff[npanels]);
  t.r_col.resize((size_t)roff[npanels]);
  t.r_cidx.resize((size_t)roff[npanels]);
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t p = 0; p < npanels; ++p) {
    const PanelOut& o = out[p];
    std::copy(o.dcols.begin(), o.dcols.end(), t.dense_cols.begin() + t.dense_ptr[p]);
    std::copy(o.d_slot.begin(), o.d_slot.end(), t.d_slot.begin() + doff[p]);
    std::copy(o.d_cidx.begin(), o.d_cidx.end(), t.d_cidx.begin() + doff[p]);
    std::copy(o.r_col.begin(), o.r_col.end(), t.r_col.begin() + roff[p]);
    std::copy(o.r_cidx.begin(), o.r_cidx.end(), t.r_cidx.begin() + roff[p]);
  }
  for (int64_t p = 0; p < npanels; ++p) {
    const int64_t q0 = p * P;
    int64_t dd = doff[p], rr = roff[p];
    for (size_t k = 0; k < out[p].dcount.size(); ++k) {
      dd += out[p].dcount[k];
      rr += out[p].rcount[k];
      t.drow_ptr[q0 + (int64_t)k + 1] = dd;
      t.rrow_ptr[q0 + (int64_t)k + 1] = rr;
    }
  }
}

// Dense nnz of the tiling of `perm` (= Tiling::n_dense() of tile_rows with the same arguments)
// without building the tiles: the AUTO round-1 decision needs only this count.
int64_t dense_count(const HostCSR& A, const std::vector<int32_t>& perm, int32_t P, int32_t dense_min) {
  const int64_t M = A.M, N = A.N;
  const int64_t npanels = (M + P - 1) / P;
  int64_t total = 0;
#pragma omp parallel reduction(+ : total)
  {
    std::vector<int32_t> cnt((size_t)N, 0);
    std::vector<int32_t> touched;
#pragma omp for schedule(dynamic, 16)
    for (int64_t p = 0; p < npanels; ++p) {
      const int64_t q0 = p * P, q1 = std::min<int64_t>(M, q0 + P);
      touched.clear();
      for (int64_t q = q0; q < q1; ++q) {
        const int64_t r = perm[q];
        for (int64_t e = A.rowptr[r]; e < A.rowptr[r + 1]; ++e) {
          const int32_t c = A.col[e];
          if (cnt[c]++ == 0) touched.push_back(c);
        }
      }
      for (int32_t c : touched) {
        if (cnt[c] >= dense_min) total += cnt[c];
        cnt[c] = 0;
      }
    }
  }
  return total;
}

// AvgSim over the non-empty remainder rows in position order, each term
// floor(2^32·inter/uni) (reading R27), exact integer sum.
void avgsim_positions(const Tiling& t, uint64_t* num, uint64_t* den) {
  const int64_t M = (int64_t)t.rrow_ptr.size() - 1;
  std::vector<int64_t> live;
  for (int64_t q = 0; q < M; ++q)
    if (t.rrow_ptr[q + 1] > t.rrow_ptr[q]) live.push_back(q);
  const int64_t L = (int64_t)live.size();
  uint64_t sum = 0;
#pragma omp parallel for reduction(+ : sum) schedule(static, 4096)
  for (int64_t k = 0; k < L - 1; ++k) {
    const int32_t* a = t.r_col.data() + t.rrow_ptr[live[k]];
    const int32_t* ae = t.r_col.data() + t.rrow_ptr[live[k] + 1];
    const int32_t* b = t.r_col.data() + t.rrow_ptr[live[k + 1]];
    const int32_t* be = t.r_col.data() + t.rrow_ptr[live[k + 1] + 1];
    const uint64_t na = ae - a, nb = be - b;
    uint64_t n = 0;
    while (a < ae && b < be) {
      if (*a == *b) {
        ++n; ++a; ++b;
      } else if (*a < *b) {
        ++a;
      } else {
        ++b;
      }
    }
    const uint64_t u = na + nb - n;
    sum += (uint64_t)(((unsigned __int128)n << 32) / u);
  }
  *num = sum;
  *den = L >= 2 ? ((uint64_t)(L - 1) << 32) : 0;
}

}  // namespace sr
