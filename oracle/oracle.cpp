// oracle.cpp -- TEST INFRASTRUCTURE ONLY (see oracle.h).
//
// The plain definition of a window-based query (§2.4),
// evaluated window by window.  Each function names the passage it follows.
// Deliberately naive: fields are decoded with memcpy at their byte offsets
// (tuples are byte records, L744-745), a window is a literal position range,
// groups live in a std::map re-created per window, sums run in increasing
// position order in fp64 (float columns) or checked int64 (int columns).
#include "oracle.h"

#include <algorithm>
#include <array>
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <map>
#include <thread>
#include <vector>

namespace {

int64_t read_int(const uint8_t *t, int32_t off, int32_t type) {
  if (type == OQ_I32) { int32_t v; std::memcpy(&v, t + off, 4); return v; }
  int64_t v; std::memcpy(&v, t + off, 8); return v;
}
double read_float(const uint8_t *t, int32_t off, int32_t type) {
  if (type == OQ_F32) { float v; std::memcpy(&v, t + off, 4); return (double)v; }
  double v; std::memcpy(&v, t + off, 8); return v;
}
bool is_float(int32_t type) { return type == OQ_F32 || type == OQ_F64; }

template <class T> bool cmp(T a, int32_t op, T b) {
  switch (op) {
    case OQ_LT: return a < b;  case OQ_LE: return a <= b;
    case OQ_GT: return a > b;  case OQ_GE: return a >= b;
    case OQ_EQ: return a == b; case OQ_NE: return a != b;
  }
  return false;
}

// σ: a conjunction of `col op const` (selection, §2.4).
bool selected(const oq_query *q, const uint8_t *t) {
  for (int p = 0; p < q->npred; ++p) {
    const oq_pred &pr = q->pred[p];
    bool ok = is_float(pr.type) ? cmp(read_float(t, pr.off, pr.type), pr.op, pr.fval)
                                : cmp(read_int(t, pr.off, pr.type), pr.op, pr.ival);
    if (!ok) return false;
  }
  return true;
}

// Per-group accumulator for the aggregation operator α (§2.4).
struct Acc {
  int64_t count = 0;
  double fsum[8] = {0};
  int64_t isum[8] = {0};
  double fmin[8], fmax[8];
  int64_t imin[8], imax[8];
  bool overflow = false;
};

struct WinOut {
  int64_t id = 0, ts = 0;
  std::vector<std::array<int64_t, 4>> keys;
  std::vector<std::array<uint64_t, 8>> vals;
  std::vector<uint8_t> bytes;  // IStream
  bool overflow = false;
};

struct Range { int64_t a, b; };

// Window extent W_j as a position range (τ is non-decreasing, L347-349).
// count: [j·l, j·l+s)  (L370-372, first window starts at t1: Fig. 2 prose L508-513)
// time : [lower_bound(T0+j·l), lower_bound(T0+j·l+s))  (reading A1 of L372-374)
Range window_range(const oq_query *q, const std::vector<int64_t> &tau, int64_t j) {
  if (q->win_kind == OQ_COUNTWIN) return {j * q->slide, j * q->slide + q->size};
  int64_t lo = q->origin + j * q->slide, hi = lo + q->size;
  int64_t a = std::lower_bound(tau.begin(), tau.end(), lo) - tau.begin();
  int64_t b = std::lower_bound(tau.begin(), tau.end(), hi) - tau.begin();
  return {a, b};
}

void eval_window(const oq_query *q, const uint8_t *tuples, const std::vector<int64_t> &tau,
                 int64_t j, WinOut &w) {
  const int64_t tb = q->tuple_bytes;
  Range r = window_range(q, tau, j);
  w.id = j;
  w.ts = (q->win_kind == OQ_COUNTWIN) ? tau[r.a] : q->origin + j * q->slide;  // reading A7
  if (q->nagg == 0) {
    // IStream (L395-400): tuples of W_j that are not part of W_{j-1} (position identity, A9).
    Range prev = (j == 0) ? Range{0, 0} : window_range(q, tau, j - 1);
    for (int64_t i = r.a; i < r.b; ++i) {
      if (i >= prev.a && i < prev.b) continue;
      const uint8_t *t = tuples + i * tb;
      if (!selected(q, t)) continue;
      for (int c = 0; c < q->nproj; ++c) {
        int w8 = (q->proj[c].type == OQ_I32 || q->proj[c].type == OQ_F32) ? 4 : 8;
        w.bytes.insert(w.bytes.end(), t + q->proj[c].off, t + q->proj[c].off + w8);
      }
    }
    return;
  }
  // RStream aggregation (L392-395), GROUP BY key = (col_k / div_k)_k (reading A17).
  std::map<std::array<int64_t, 4>, Acc> groups;
  for (int64_t i = r.a; i < r.b; ++i) {
    const uint8_t *t = tuples + i * tb;
    if (!selected(q, t)) continue;  // σ inside the window (reading A5)
    std::array<int64_t, 4> key{0, 0, 0, 0};
    for (int k = 0; k < q->nkeys; ++k)
      key[k] = read_int(t, q->key[k].off, q->key[k].type) / q->key[k].div;
    auto it = groups.find(key);
    if (it == groups.end()) {
      Acc fresh;
      for (int a = 0; a < q->nagg; ++a) {
        fresh.fmin[a] = 0; fresh.fmax[a] = 0; fresh.imin[a] = 0; fresh.imax[a] = 0;
      }
      it = groups.emplace(key, fresh).first;
    }
    Acc &acc = it->second;
    bool first = (acc.count == 0);
    acc.count += 1;
    for (int a = 0; a < q->nagg; ++a) {
      const oq_agg &ag = q->agg[a];
      if (ag.fn == OQ_COUNT) continue;
      if (is_float(ag.type)) {
        double x = read_float(t, ag.off, ag.type);
        acc.fsum[a] += x;                         // increasing i, fp64 (reading A12)
        if (first || x < acc.fmin[a]) acc.fmin[a] = x;
        if (first || x > acc.fmax[a]) acc.fmax[a] = x;
      } else {
        int64_t x = read_int(t, ag.off, ag.type);
        if (__builtin_add_overflow(acc.isum[a], x, &acc.isum[a])) acc.overflow = true;
        if (first || x < acc.imin[a]) acc.imin[a] = x;
        if (first || x > acc.imax[a]) acc.imax[a] = x;
      }
    }
  }
  for (auto &kv : groups) {  // std::map: ascending key order (reading A8)
    const Acc &acc = kv.second;
    if (acc.overflow) w.overflow = true;
    std::array<uint64_t, 8> v{};
    std::array<double, 8> fv{};
    std::array<int64_t, 8> iv{};
    std::array<bool, 8> isf{};
    for (int a = 0; a < q->nagg; ++a) {
      const oq_agg &ag = q->agg[a];
      bool fcol = is_float(ag.type);
      switch (ag.fn) {
        case OQ_COUNT: iv[a] = acc.count; isf[a] = false; break;
        case OQ_SUM: if (fcol) { fv[a] = acc.fsum[a]; isf[a] = true; }
                     else { iv[a] = acc.isum[a]; isf[a] = false; } break;
        case OQ_AVG: fv[a] = (fcol ? acc.fsum[a] : (double)acc.isum[a]) / (double)acc.count;
                     isf[a] = true; break;   // reading A11
        case OQ_MIN: if (fcol) { fv[a] = acc.fmin[a]; isf[a] = true; }
                     else { iv[a] = acc.imin[a]; isf[a] = false; } break;
        case OQ_MAX: if (fcol) { fv[a] = acc.fmax[a]; isf[a] = true; }
                     else { iv[a] = acc.imax[a]; isf[a] = false; } break;
      }
      if (isf[a]) std::memcpy(&v[a], &fv[a], 8); else std::memcpy(&v[a], &iv[a], 8);
    }
    // HAVING: selection over the finalised window results (L1291-1292, L1335-1336; A16).
    bool keep = true;
    for (int h = 0; h < q->nhave && keep; ++h) {
      const oq_have &hv = q->have[h];
      keep = isf[hv.agg] ? cmp(fv[hv.agg], hv.op, hv.fval) : cmp(iv[hv.agg], hv.op, hv.ival);
    }
    if (!keep) continue;
    w.keys.push_back(kv.first);
    w.vals.push_back(v);
  }
}

int64_t closed_windows(const oq_query *q, const std::vector<int64_t> &tau, int64_t n,
                       int64_t wm, int32_t has_wm) {
  if (q->win_kind == OQ_COUNTWIN) {            // complete windows only (reading A3)
    if (n < q->size) return 0;
    return (n - q->size) / q->slide + 1;
  }
  if (!has_wm) {
    if (n == 0) return 0;
    wm = tau[n - 1] + 1;
  }
  // j closed iff T0 + j·l + s <= wm
  int64_t span = wm - q->origin - q->size;
  if (span < 0) return 0;
  return span / q->slide + 1;
}

int validate(const oq_query *q, const uint8_t *tuples, int64_t n, std::vector<int64_t> &tau) {
  if (q->size < 1 || q->slide < 1 || q->tuple_bytes < 8) return OQ_EINVAL;
  if (q->nagg > 8 || q->nkeys > 4 || q->npred > 64 || q->nproj > 16 || q->nhave > 8) return OQ_EINVAL;
  for (int k = 0; k < q->nkeys; ++k) if (q->key[k].div == 0) return OQ_EINVAL;
  tau.resize(n);
  for (int64_t i = 0; i < n; ++i) {
    std::memcpy(&tau[i], tuples + i * q->tuple_bytes + q->ts_off, 8);
    if (tau[i] < 0) return OQ_EINVAL;                          // reading A24
    if (i > 0 && tau[i] < tau[i - 1]) return OQ_EORDER;        // L347-349
  }
  return OQ_OK;
}

}  // namespace

extern "C" int64_t oq_num_windows(const oq_query *q, const uint8_t *tuples, int64_t n,
                                  int64_t watermark, int32_t has_wm) {
  std::vector<int64_t> tau;
  if (validate(q, tuples, n, tau) != OQ_OK) return -1;
  return closed_windows(q, tau, n, watermark, has_wm);
}

extern "C" int32_t oq_run(const oq_query *q, const uint8_t *tuples, int64_t n,
                          int64_t watermark, int32_t has_wm,
                          const int64_t *window_ids, int64_t nids, int32_t nthreads,
                          oq_result *out) {
  std::memset(out, 0, sizeof(*out));
  std::vector<int64_t> tau;
  int err = validate(q, tuples, n, tau);
  if (err != OQ_OK) { out->error = err; return err; }
  int64_t nw = closed_windows(q, tau, n, watermark, has_wm);
  std::vector<int64_t> ids;
  if (window_ids) {
    ids.assign(window_ids, window_ids + nids);
    for (int64_t j : ids) if (j < 0 || j >= nw) { out->error = OQ_EINVAL; return OQ_EINVAL; }
  } else {
    ids.resize(nw);
    for (int64_t j = 0; j < nw; ++j) ids[j] = j;
  }
  std::vector<WinOut> wins(ids.size());
  if (nthreads < 1) nthreads = 1;
  std::atomic<int64_t> next{0};
  auto worker = [&]() {
    for (;;) {
      int64_t k = next.fetch_add(1);
      if (k >= (int64_t)ids.size()) break;
      eval_window(q, tuples, tau, ids[k], wins[k]);
    }
  };
  if (nthreads == 1) worker();
  else {
    std::vector<std::thread> th;
    for (int t = 0; t < nthreads; ++t) th.emplace_back(worker);
    for (auto &t : th) t.join();
  }
  // RStream / IStream concatenation in window order (L392-400).
  int64_t nrows = 0, nbytes = 0;
  for (auto &w : wins) { nrows += (int64_t)w.keys.size(); nbytes += (int64_t)w.bytes.size(); }
  out->nwin = (int64_t)wins.size();
  out->win_id = (int64_t *)std::malloc(sizeof(int64_t) * (wins.size() + 1));
  out->win_ts = (int64_t *)std::malloc(sizeof(int64_t) * (wins.size() + 1));
  out->win_nrows = (int64_t *)std::malloc(sizeof(int64_t) * (wins.size() + 1));
  out->win_rowoff = (int64_t *)std::malloc(sizeof(int64_t) * (wins.size() + 1));
  out->nrows = nrows;
  out->keys = (int64_t *)std::malloc(sizeof(int64_t) * (nrows * (q->nkeys > 0 ? q->nkeys : 1) + 1));
  out->vals = (uint64_t *)std::malloc(sizeof(uint64_t) * (nrows * (q->nagg > 0 ? q->nagg : 1) + 1));
  out->out_bytes = nbytes;
  out->out = (uint8_t *)std::malloc(nbytes + 1);
  int64_t rb = 0;
  for (int c = 0; c < q->nproj; ++c)
    rb += (q->proj[c].type == OQ_I32 || q->proj[c].type == OQ_F32) ? 4 : 8;
  out->row_bytes = rb;
  for (int a = 0; a < q->nagg; ++a) {
    const oq_agg &ag = q->agg[a];
    out->val_is_float[a] = (ag.fn == OQ_AVG) || (ag.fn != OQ_COUNT && is_float(ag.type));
  }
  int64_t r = 0, b = 0;
  bool overflow = false;
  for (size_t k = 0; k < wins.size(); ++k) {
    WinOut &w = wins[k];
    overflow |= w.overflow;
    out->win_id[k] = w.id;
    out->win_ts[k] = w.ts;
    out->win_nrows[k] = (q->nagg > 0) ? (int64_t)w.keys.size() : (int64_t)(w.bytes.size() / (rb ? rb : 1));
    out->win_rowoff[k] = (q->nagg > 0) ? r : b / (rb ? rb : 1);
    for (size_t i = 0; i < w.keys.size(); ++i, ++r) {
      for (int kk = 0; kk < q->nkeys; ++kk) out->keys[r * q->nkeys + kk] = w.keys[i][kk];
      for (int a = 0; a < q->nagg; ++a) out->vals[r * q->nagg + a] = w.vals[i][a];
    }
    if (!w.bytes.empty()) std::memcpy(out->out + b, w.bytes.data(), w.bytes.size());
    b += (int64_t)w.bytes.size();
  }
  if (overflow) out->error = OQ_EOVERFLOW;
  return out->error;
}

extern "C" void oq_free(oq_result *r) {
  std::free(r->win_id); std::free(r->win_ts); std::free(r->win_nrows); std::free(r->win_rowoff);
  std::free(r->keys); std::free(r->vals); std::free(r->out);
  std::memset(r, 0, sizeof(*r));
}

// ---------------------------------------------------------------------------
// Windowed θ-join (oracle.h): window j = W1_j ⋈θ W2_j, both count windows
// [j·l, j·l+s); every pair tested literally, in (a, b) order.
namespace {
bool jpred_ok(const oq_join *q, const uint8_t *a, const uint8_t *b) {
  for (int p = 0; p < q->npred; ++p) {
    const oq_jpred &pr = q->pred[p];
    bool ok;
    if (is_float(pr.type1) || is_float(pr.type2)) {
      const double x = is_float(pr.type1) ? read_float(a, pr.off1, pr.type1) : (double)read_int(a, pr.off1, pr.type1);
      const double y = is_float(pr.type2) ? read_float(b, pr.off2, pr.type2) : (double)read_int(b, pr.off2, pr.type2);
      ok = cmp(x, pr.op, y);
    } else {
      ok = cmp(read_int(a, pr.off1, pr.type1), pr.op, read_int(b, pr.off2, pr.type2));
    }
    if (!ok) return false;
  }
  return true;
}
int col_width(int32_t type) { return (type == OQ_I32 || type == OQ_F32) ? 4 : 8; }
}  // namespace

extern "C" int32_t oq_join_run(const oq_join *q, const uint8_t *t1, int64_t n1, const uint8_t *t2, int64_t n2,
                               int32_t nthreads, oq_result *out) {
  std::memset(out, 0, sizeof(*out));
  if (q->size < 1 || q->slide < 1 || q->npred < 0 || q->npred > 64 || q->nproj1 > 16 || q->nproj2 > 16) {
    out->error = OQ_EINVAL;
    return OQ_EINVAL;
  }
  const int64_t n = n1 < n2 ? n1 : n2;
  const int64_t nw = n >= q->size ? (n - q->size) / q->slide + 1 : 0;
  int64_t rb = 0;
  for (int c = 0; c < q->nproj1; ++c) rb += col_width(q->proj1[c].type);
  for (int c = 0; c < q->nproj2; ++c) rb += col_width(q->proj2[c].type);
  std::vector<std::vector<uint8_t>> wins((size_t)nw);
  std::atomic<int64_t> next{0};
  auto worker = [&]() {
    for (;;) {
      const int64_t j = next.fetch_add(1);
      if (j >= nw) break;
      std::vector<uint8_t> &o = wins[(size_t)j];
      for (int64_t a = j * q->slide; a < j * q->slide + q->size; ++a) {
        const uint8_t *ta = t1 + a * q->tuple_bytes1;
        for (int64_t b = j * q->slide; b < j * q->slide + q->size; ++b) {
          const uint8_t *tb = t2 + b * q->tuple_bytes2;
          if (!jpred_ok(q, ta, tb)) continue;
          for (int c = 0; c < q->nproj1; ++c)
            o.insert(o.end(), ta + q->proj1[c].off, ta + q->proj1[c].off + col_width(q->proj1[c].type));
          for (int c = 0; c < q->nproj2; ++c)
            o.insert(o.end(), tb + q->proj2[c].off, tb + q->proj2[c].off + col_width(q->proj2[c].type));
        }
      }
    }
  };
  if (nthreads < 1) nthreads = 1;
  if (nthreads == 1) worker();
  else {
    std::vector<std::thread> th;
    for (int t = 0; t < nthreads; ++t) th.emplace_back(worker);
    for (auto &t : th) t.join();
  }
  int64_t nbytes = 0;
  for (auto &w : wins) nbytes += (int64_t)w.size();
  out->nwin = nw;
  out->win_id = (int64_t *)std::malloc(sizeof(int64_t) * (nw + 1));
  out->win_ts = (int64_t *)std::malloc(sizeof(int64_t) * (nw + 1));
  out->win_nrows = (int64_t *)std::malloc(sizeof(int64_t) * (nw + 1));
  out->win_rowoff = (int64_t *)std::malloc(sizeof(int64_t) * (nw + 1));
  out->keys = (int64_t *)std::malloc(8);
  out->vals = (uint64_t *)std::malloc(8);
  out->out_bytes = nbytes;
  out->out = (uint8_t *)std::malloc(nbytes + 1);
  out->row_bytes = rb;
  int64_t off = 0;
  for (int64_t j = 0; j < nw; ++j) {
    int64_t ts;
    std::memcpy(&ts, t1 + j * q->slide * q->tuple_bytes1 + q->ts_off1, 8);   // reading A7
    out->win_id[j] = j;
    out->win_ts[j] = ts;
    out->win_nrows[j] = rb ? (int64_t)wins[(size_t)j].size() / rb : 0;
    out->win_rowoff[j] = rb ? off / rb : 0;
    if (!wins[(size_t)j].empty()) std::memcpy(out->out + off, wins[(size_t)j].data(), wins[(size_t)j].size());
    off += (int64_t)wins[(size_t)j].size();
  }
  out->nrows = rb ? nbytes / rb : 0;
  return OQ_OK;
}
