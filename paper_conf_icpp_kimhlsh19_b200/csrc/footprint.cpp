// footprint.cpp — the CATT footprint analyser (host only), steps a1-a5.
//
//   a1  Eq 1-3 resident CTAs per SM, plus the grid bound
//       ceil(grid / #SM) that Table 3's ATAX baseline (8,4) under
//       <<<80*4, 256>>> requires; Eq 4 the
//       smallest shared-memory option that holds them, and the L1D it leaves.
//   a2  Eq 5-6: reuse iff |C_i| * elem_bytes < line, at a level
//       that iterates (trip >= 2); loops without any reuse are not throttled
//       ("for loops where cache locality presents").
//   a3  Eq 7: lines per warp per memory instruction.
//   a4  Eq 8: footprint. Paper mode = the printed per-warp sum;
//       union mode (B200 default) = distinct lines of the co-resident warps,
//       enumerated lane by lane ("we examine every address accessed by each
//       thread in a warp"), maximised over the co-resident CTA window,
//       the Fig 4 warp group and the phase of the innermost loop.
//   a5  Eq 9 (order P:357): warp level over the divisors
//       N of #Warps_TB, then CTA level with one warp per CTA, else give up
//       (P:395).
// DESIGN.md "Readings" lists every interpretation (R1-R17) this file takes.
#include <algorithm>
#include <climits>
#include <cstdint>
#include <cstring>
#include <map>
#include <unordered_set>
#include <vector>

#include "../../include/catt.h"

namespace {

constexpr int64_t kMaxWindow = int64_t(1) << 20;

int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
int64_t round_up(int64_t a, int64_t b) { return ceil_div(a, b) * b; }
int64_t floor_div(int64_t a, int64_t b) {
  int64_t q = a / b;
  if ((a % b != 0) && ((a < 0) != (b < 0))) --q;
  return q;
}
int64_t iabs(int64_t v) { return v < 0 ? -v : v; }

struct Occ {
  int32_t W = 0, T = 0, carveout_kb = 0;
  int64_t l1d = 0;
};

// a1: Eq 1-4.
catt_status occupancy(const catt_loop_desc& d, const catt_hw& hw, Occ* o) {
  const int64_t threads = int64_t(d.block[0]) * d.block[1] * d.block[2];
  const int32_t W = int32_t(ceil_div(threads, hw.warp_size));
  const bool paper = d.mode == CATT_MODE_PAPER;
  int64_t smem_cta = paper ? d.smem_per_cta
                           : round_up(int64_t(d.smem_per_cta) + hw.reserved_smem_cta, hw.smem_alloc_unit);
  int32_t max_carve = 0;
  for (int i = 0; i < hw.n_carveouts; ++i) max_carve = std::max(max_carve, hw.carveout_kb[i]);
  int64_t T = INT64_MAX;
  if (smem_cta > 0) T = std::min(T, int64_t(max_carve) * 1024 / smem_cta);        // Eq 1
  if (d.regs_per_thread > 0) {                                                    // Eq 2
    if (paper) {
      T = std::min(T, int64_t(hw.regs_sm) / (int64_t(d.regs_per_thread) * threads));
    } else {
      int64_t per_warp = round_up(int64_t(d.regs_per_thread) * hw.warp_size, hw.reg_alloc_unit);
      int64_t warps = 4 * ((int64_t(hw.regs_sm) / 4) / per_warp);                 // 4 SM sub-partitions
      T = std::min(T, warps / W);
    }
  }
  T = std::min(T, int64_t(std::min(hw.max_ctas_sm, hw.max_warps_sm / W)));        // #TB_HW
  const int64_t nblocks = d.grid[0] * d.grid[1] * d.grid[2];
  T = std::min(T, ceil_div(nblocks, hw.num_sms));                                 // grid bound
  if (T < 1) return CATT_EINVAL;
  int idx = -1;
  if (d.force_carveout_kb >= 0) {
    for (int i = 0; i < hw.n_carveouts; ++i)
      if (hw.carveout_kb[i] == d.force_carveout_kb) idx = i;
    if (idx < 0) return CATT_EINVAL;
    if (smem_cta > 0) T = std::min(T, int64_t(hw.carveout_kb[idx]) * 1024 / smem_cta);
    if (T < 1) return CATT_EINVAL;
  } else {
    const int64_t need = T * smem_cta;                                            // Eq 4
    for (int i = 0; i < hw.n_carveouts && idx < 0; ++i)
      if (int64_t(hw.carveout_kb[i]) * 1024 >= need) idx = i;
    if (idx < 0) return CATT_EINVAL;
  }
  o->W = W;
  o->T = int32_t(T);
  o->carveout_kb = hw.carveout_kb[idx];
  o->l1d = hw.l1d_bytes[idx];
  return CATT_OK;
}

struct G3 {
  int64_t v[3];
};

// Global coordinates of the valid lanes of warp w of CTA b (x fastest).
std::vector<G3> lane_gids(const catt_loop_desc& d, int64_t b, int32_t w, int32_t warp_size) {
  std::vector<G3> out;
  const int64_t bx = d.block[0], by = d.block[1], bz = d.block[2];
  const int64_t threads = bx * by * bz;
  const int64_t cb[3] = {b % d.grid[0], (b / d.grid[0]) % d.grid[1], b / (d.grid[0] * d.grid[1])};
  for (int lane = 0; lane < warp_size; ++lane) {
    const int64_t t = int64_t(w) * warp_size + lane;
    if (t >= threads) break;
    const int64_t ct[3] = {t % bx, (t / bx) % by, t / (bx * by)};
    G3 g;
    bool ok = true;
    for (int k = 0; k < 3; ++k) {
      g.v[k] = cb[k] * d.block[k] + ct[k];
      if (d.extent[k] > 0 && g.v[k] >= d.extent[k]) ok = false;
    }
    if (ok) out.push_back(g);
  }
  return out;
}

struct Window {
  bool per_phase = true;                 // evaluate at (0, .., 0, k)
  std::vector<std::vector<int64_t>> its; // fixed window of an outer-level reuse
};

catt_status make_window(const catt_ref& r, const catt_loop_desc& d, int32_t line, Window* w) {
  const int n = d.n_loops;
  w->per_phase = true;
  w->its.clear();
  if (n == 0) return CATT_OK;
  const int L = n - 1;
  if (iabs(r.c_iter[L]) * r.elem_bytes < line) return CATT_OK;                 // consecutive reuse
  for (int k = L - 1; k >= 0; --k) {
    if (iabs(r.c_iter[k]) * r.elem_bytes < line) {                              // reuse across level k
      int64_t size = 1;
      for (int q = k + 1; q < n; ++q) {
        size *= d.trip[q];
        if (size > kMaxWindow) return CATT_EUNSUPPORTED;
      }
      std::vector<int64_t> it(n, 0);
      for (int64_t c = 0; c < size; ++c) {
        int64_t rem = c;
        for (int q = n - 1; q > k; --q) {
          it[q] = rem % d.trip[q];
          rem /= d.trip[q];
        }
        w->its.push_back(it);
      }
      w->per_phase = false;
      return CATT_OK;
    }
  }
  return CATT_OK;                                                               // no reuse
}

inline uint64_t line_key(int32_t array_id, int64_t line) {
  return (uint64_t(uint32_t(array_id)) << 44) ^ uint64_t(line & ((int64_t(1) << 44) - 1));
}

void add_lines(const catt_ref& r, const std::vector<G3>& gids, const std::vector<int64_t>& it, int n_loops,
               int32_t line, std::unordered_set<uint64_t>* s) {
  const bool irr = (r.flags & CATT_REF_IRREGULAR) != 0;
  const int64_t cg[3] = {irr ? 1 : r.c_gid[0], irr ? 0 : r.c_gid[1], irr ? 0 : r.c_gid[2]};
  int64_t itoff = 0;
  for (int k = 0; k < n_loops; ++k) itoff += r.c_iter[k] * it[k];
  for (const G3& g : gids) {
    const int64_t idx = r.base + cg[0] * g.v[0] + cg[1] * g.v[1] + cg[2] * g.v[2] + itoff;
    s->insert(line_key(r.array_id, floor_div(idx * r.elem_bytes, line)));
  }
}

// a3 paper mode: REQ_warp (Eq 7), generalised to elem_bytes (R2).
int64_t req_warp_paper(const catt_ref& r, const catt_loop_desc& d, const catt_hw& hw) {
  if (r.flags & CATT_REF_NOT_L1) return 0;
  const int64_t ws = hw.warp_size, line = hw.line_bytes;
  if (d.block[0] % ws == 0 || (r.flags & CATT_REF_IRREGULAR)) {
    const int64_t c = (r.flags & CATT_REF_IRREGULAR) ? 1 : iabs(r.c_gid[0]);
    if (c == 0) return 1;
    return std::min(ws, ceil_div(ws * c * r.elem_bytes, line));
  }
  // warps span several rows of a multi-dimensional block: examine every address
  std::unordered_set<uint64_t> s;
  std::vector<int64_t> it0(d.n_loops, 0);
  add_lines(r, lane_gids(d, 0, 0, hw.warp_size), it0, d.n_loops, hw.line_bytes, &s);
  return std::max<int64_t>(1, int64_t(s.size()));
}

class Model {
 public:
  Model(const catt_loop_desc& d, const catt_hw& hw, const Occ& o) : d_(d), hw_(hw), o_(o) {}

  catt_status init() {
    line_ = hw_.line_bytes;
    paper_ = d_.mode == CATT_MODE_PAPER;
    locality_ = false;
    for (int i = 0; i < d_.n_refs; ++i) {
      const catt_ref& r = d_.refs[i];
      if (r.flags & CATT_REF_NOT_L1) continue;
      for (int k = 0; k < d_.n_loops; ++k)
        if (iabs(r.c_iter[k]) * r.elem_bytes < line_ && d_.trip[k] >= 2) locality_ = true;
    }
    if (paper_) {
      req_ = 0;
      for (int i = 0; i < d_.n_refs; ++i) req_ += req_warp_paper(d_.refs[i], d_, hw_);
      lines_per_warp_iter_ = reuse_span_ = req_;
      return CATT_OK;
    }
    bool any_phase = false;
    for (int i = 0; i < d_.n_refs; ++i) {
      const catt_ref& r = d_.refs[i];
      if (r.flags & (CATT_REF_NOT_L1 | CATT_REF_STORE)) continue;
      Window w;
      catt_status st = make_window(r, d_, line_, &w);
      if (st != CATT_OK) return st;
      any_phase = any_phase || w.per_phase;
      refs_.push_back(r);
      win_.push_back(std::move(w));
    }
    const int64_t nblocks = d_.grid[0] * d_.grid[1] * d_.grid[2];
    for (int64_t k = 0; k < o_.T; ++k)
      if (k * hw_.num_sms < nblocks) blocks_.push_back(k * hw_.num_sms);
    phases_ = (any_phase && d_.n_loops > 0) ? std::min<int64_t>(d_.trip[d_.n_loops - 1], line_ / 4) : 1;
    // lines touched by warp 0 of CTA 0 in iteration 0, per memory instruction
    const std::vector<G3> g00 = lane_gids(d_, 0, 0, hw_.warp_size);
    const std::vector<int64_t> it0(d_.n_loops, 0);
    lines_per_warp_iter_ = 0;
    // B200 guard (R18, R23): some reused reference is memory-divergent
    // (>= divergent_lines lines per warp request), re-touches its line often
    // enough (>= min_retouch times per thread) and keeps reusing for long
    // enough (a reuse loop of >= min_reuse_trip iterations)
    divergent_ = hw_.divergent_lines <= 0 && hw_.min_retouch <= 0 && hw_.min_reuse_trip <= 0 && hw_.max_stream_pct <= 0;
    for (const catt_ref& r : refs_) {
      std::unordered_set<uint64_t> s;
      add_lines(r, g00, it0, d_.n_loops, line_, &s);
      lines_per_warp_iter_ += int64_t(s.size());
      bool reuse = false;
      int64_t retouch = 0, rtrip = 0;
      for (int k = 0; k < d_.n_loops; ++k)
        if (iabs(r.c_iter[k]) * r.elem_bytes < line_ && d_.trip[k] >= 2) {
          reuse = true;
          const int64_t per_line = r.c_iter[k] == 0 ? d_.trip[k]
                                                     : std::min<int64_t>(d_.trip[k], line_ / (iabs(r.c_iter[k]) * r.elem_bytes));
          retouch = std::max(retouch, per_line);
          rtrip = std::max(rtrip, d_.trip[k]);
        }
      // R32: a divergent load whose lines every warp of the CTA requests too
      // (warp 1 touches the same lines as warp 0) is served to the CTA's
      // warps by one fill: it does not make the loop divergent
      bool cta_shared = false;
      if (hw_.private_streams > 0 && o_.W >= 2 && int64_t(s.size()) >= hw_.divergent_lines) {
        std::unordered_set<uint64_t> s1;
        add_lines(r, lane_gids(d_, 0, 1, hw_.warp_size), it0, d_.n_loops, line_, &s1);
        cta_shared = s1 == s;
      }
      if (reuse && !cta_shared && int64_t(s.size()) >= hw_.divergent_lines && retouch >= hw_.min_retouch &&
          rtrip >= hw_.min_reuse_trip) {
        divergent_ = true;
        ++streams_;                    // R29: one more memory-divergent reused load
      }
    }
    // R24: no throttle when more than max_stream_pct % of a lane's bytes per
    // iteration belong to streams L1 cannot serve again (stores, loads
    // without reuse): those need the memory-level parallelism a throttle removes
    if (hw_.max_stream_pct > 0) {
      int64_t total = 0, stream = 0;
      for (int i = 0; i < d_.n_refs; ++i) {
        const catt_ref& r = d_.refs[i];
        if (r.flags & CATT_REF_NOT_L1) continue;
        total += r.elem_bytes;
        bool reuse = false;
        for (int k = 0; k < d_.n_loops; ++k)
          if (iabs(r.c_iter[k]) * r.elem_bytes < line_ && d_.trip[k] >= 2) reuse = true;
        if ((r.flags & CATT_REF_STORE) || !reuse) stream += r.elem_bytes;
      }
      if (100 * stream > int64_t(hw_.max_stream_pct) * total) divergent_ = false;
    }
    reuse_span_ = int64_t(retained(0, 0, 0).size());
    return CATT_OK;
  }

  const std::vector<uint64_t>& retained(size_t bi, int32_t w, int64_t k) {
    const uint64_t key = (uint64_t(bi) << 40) | (uint64_t(w) << 20) | uint64_t(k);
    auto it = cache_.find(key);
    if (it != cache_.end()) return it->second;
    const int64_t b = blocks_.empty() ? 0 : blocks_[bi];
    const std::vector<G3> gids = lane_gids(d_, b, w, hw_.warp_size);
    std::unordered_set<uint64_t> s;
    std::vector<int64_t> ph(d_.n_loops, 0);
    if (d_.n_loops > 0) ph[d_.n_loops - 1] = k;
    for (size_t i = 0; i < refs_.size(); ++i) {
      if (win_[i].per_phase) {
        add_lines(refs_[i], gids, ph, d_.n_loops, line_, &s);
      } else {
        for (const auto& itv : win_[i].its) add_lines(refs_[i], gids, itv, d_.n_loops, line_, &s);
      }
    }
    std::vector<uint64_t> v(s.begin(), s.end());
    return cache_.emplace(key, std::move(v)).first->second;
  }

  // Footprint in lines with a active warps per CTA and m CTAs per SM.
  int64_t F(int32_t a, int32_t m) {
    if (paper_) return req_ * a * m;                                             // Eq 8 / Eq 9
    int64_t best = 0;
    const int64_t nb = int64_t(blocks_.size());
    const int64_t n_windows = std::max<int64_t>(1, nb - m + 1);
    const int32_t groups = int32_t(ceil_div(o_.W, a));
    for (int64_t s0 = 0; s0 < n_windows; ++s0) {
      for (int32_t g = 0; g < groups; ++g) {
        for (int64_t k = 0; k < phases_; ++k) {
          std::unordered_set<uint64_t> u;
          for (int64_t bi = s0; bi < std::min(nb, s0 + m); ++bi)
            for (int32_t w = g * a; w < std::min(o_.W, g * a + a); ++w) {
              const auto& r = retained(size_t(bi), w, k);
              u.insert(r.begin(), r.end());
            }
          best = std::max(best, int64_t(u.size()));
        }
      }
    }
    return best;
  }

  bool fits(int64_t lines) const { return lines * line_ <= o_.l1d; }

  bool locality_ = false;
  bool divergent_ = true;  // some reused reference is memory-divergent (B200 guard)
  int32_t streams_ = 0;    // how many (R29)
  int64_t lines_per_warp_iter_ = 0, reuse_span_ = 0;

 private:
  const catt_loop_desc& d_;
  const catt_hw& hw_;
  const Occ& o_;
  int32_t line_ = 128;
  bool paper_ = false;
  int64_t req_ = 0, phases_ = 1;
  std::vector<catt_ref> refs_;
  std::vector<Window> win_;
  std::vector<int64_t> blocks_;
  std::map<uint64_t, std::vector<uint64_t>> cache_;
};

catt_status validate(const catt_loop_desc* d, const catt_hw* hw) {
  if (!d || !hw) return CATT_EINVAL;
  if (d->n_refs < 0 || d->n_refs > 64 || (d->n_refs > 0 && !d->refs)) return CATT_EINVAL;
  if (d->n_loops < 0 || d->n_loops > CATT_MAX_LOOPS) return CATT_EINVAL;
  for (int k = 0; k < d->n_loops; ++k)
    if (d->trip[k] < 1) return CATT_EINVAL;
  int64_t threads = 1;
  for (int k = 0; k < 3; ++k) {
    if (d->block[k] < 1 || d->grid[k] < 1 || d->extent[k] < 0) return CATT_EINVAL;
    threads *= d->block[k];
  }
  if (threads > 1024) return CATT_EINVAL;
  if (d->mode != CATT_MODE_UNION && d->mode != CATT_MODE_PAPER) return CATT_EINVAL;
  if (d->regs_per_thread < 0 || d->smem_per_cta < 0) return CATT_EINVAL;
  for (int i = 0; i < d->n_refs; ++i) {
    const int e = d->refs[i].elem_bytes;
    if (e != 1 && e != 2 && e != 4 && e != 8 && e != 16 && e != 32) return CATT_EINVAL;
    if (d->refs[i].array_id < 0) return CATT_EINVAL;
  }
  if (hw->warp_size != 32 || hw->num_sms < 1 || hw->max_warps_sm < 1 || hw->max_ctas_sm < 1) return CATT_EINVAL;
  if (hw->line_bytes < 4 || hw->n_carveouts < 1 || hw->n_carveouts > CATT_MAX_CARVEOUTS) return CATT_EINVAL;
  if (hw->smem_alloc_unit < 1 || hw->reg_alloc_unit < 1 || hw->regs_sm < 1) return CATT_EINVAL;
  if (hw->min_warps_sm < 0 || hw->divergent_lines < 0 || hw->min_retouch < 0 || hw->min_reuse_trip < 0 ||
      hw->max_stream_pct < 0 || hw->max_stream_pct > 100 || hw->stream_floor < 0 || hw->private_streams < 0)
    return CATT_EINVAL;
  for (int i = 1; i < hw->n_carveouts; ++i)
    if (hw->carveout_kb[i] <= hw->carveout_kb[i - 1]) return CATT_EINVAL;
  return CATT_OK;
}

}  // namespace

extern "C" catt_status catt_footprint(const catt_loop_desc* desc, const catt_hw* hw, catt_footprint_result* out) {
  if (!out) return CATT_EINVAL;
  catt_status st = validate(desc, hw);
  if (st != CATT_OK) return st;
  Occ o;
  st = occupancy(*desc, *hw, &o);
  if (st != CATT_OK) return st;
  Model M(*desc, *hw, o);
  st = M.init();
  if (st != CATT_OK) return st;
  const int32_t W = o.W, T = o.T;
  const int64_t full = M.F(W, T);
  catt_footprint_result r;
  std::memset(&r, 0, sizeof(r));
  r.lines_per_warp_iter = M.lines_per_warp_iter_;
  r.reuse_span = M.reuse_span_;
  r.footprint_lines_full = full;
  r.l1d_bytes = o.l1d;
  r.base_warps = W;
  r.base_ctas = T;
  r.carveout_kb = o.carveout_kb;
  auto done = [&](int32_t a, int32_t m, int64_t lines, int32_t flag) {
    r.active_warps = a;
    r.active_ctas = m;
    r.footprint_lines = lines;
    r.footprint_bytes = lines * hw->line_bytes;
    r.flags = flag;
    *out = r;
    return CATT_OK;
  };
  if (M.fits(full) || !M.locality_) return done(W, T, full, CATT_FIT_NONE_NEEDED);
  const bool paper = desc->mode == CATT_MODE_PAPER;
  const bool guards =
      !paper && (hw->min_warps_sm > 0 || hw->divergent_lines > 0 || hw->min_retouch > 0 || hw->min_reuse_trip > 0 ||
                 hw->max_stream_pct > 0);
  if (guards) {
    // B200 rule (R18, R19): only memory-divergent loops; every (a, m) pair
    // with a | W, m <= T, by active warps per SM descending, ties -> fewer
    // CTAs with more warps each; never below min_warps_sm; if nothing at or
    // above the floor fits, the most throttled pair that respects it.
    if (!M.divergent_) return done(W, T, full, CATT_FIT_NONE_NEEDED | CATT_FIT_GUARDED);
    int32_t floor_w = std::max(0, hw->min_warps_sm);
    // R29: with one CTA per SM, S divergent streams per warp keep the lines
    // in flight of S times as many warps: the floor scales by 1/S
    if (hw->stream_floor > 0 && T == 1 && M.streams_ >= 2) floor_w = (floor_w + M.streams_ - 1) / M.streams_;
    std::vector<std::pair<int32_t, int32_t>> cands;
    for (int32_t a = W; a >= 1; --a) {
      if (W % a) continue;
      for (int32_t m = T; m >= 1; --m)
        if (!(a == W && m == T) && a * m >= floor_w) cands.push_back({a, m});
    }
    std::stable_sort(cands.begin(), cands.end(), [](const std::pair<int32_t, int32_t>& x,
                                                    const std::pair<int32_t, int32_t>& y) {
      if (x.first * x.second != y.first * y.second) return x.first * x.second > y.first * y.second;
      return x.first > y.first;
    });
    auto flag_of = [&](int32_t a, int32_t m) {
      return (a < W ? CATT_FIT_WARP : 0) | (m < T ? CATT_FIT_CTA : 0);
    };
    for (const auto& c2 : cands) {
      const int64_t f = M.F(c2.first, c2.second);
      if (M.fits(f)) return done(c2.first, c2.second, f, flag_of(c2.first, c2.second));
    }
    if (cands.empty()) return done(W, T, full, CATT_FIT_NONE_NEEDED | CATT_FIT_GUARDED);
    // most throttled allowed: fewest warps, then the largest a among those
    std::pair<int32_t, int32_t> last = cands.back();
    for (const auto& c2 : cands)
      if (c2.first * c2.second == last.first * last.second && c2.first > last.first) last = c2;
    // R27 (cta_fallback): with several CTAs per SM, cap whole CTAs instead,
    // (W, m) with the smallest m such that floor <= W m <= 2 floor (held-out
    // sets 6 and 7: a CTA cap beats gating warps at a similar warp count)
    if (hw->cta_fallback > 0 && T >= 2)
      for (int32_t m = 1; m <= T; ++m)
        if (int64_t(W) * m >= floor_w && int64_t(W) * m <= 2 * int64_t(floor_w)) {
          if (m == T) return done(W, T, full, CATT_FIT_NONE_NEEDED | CATT_FIT_GUARDED);
          last = {W, m};
          break;
        }
    return done(last.first, last.second, M.F(last.first, last.second),
                flag_of(last.first, last.second) | CATT_FIT_GUARDED);
  }
  for (int32_t N = 2; N <= W; ++N) {                     // Eq 9: warp level first
    if (W % N) continue;
    const int64_t f = M.F(W / N, T);
    if (M.fits(f)) return done(W / N, T, f, CATT_FIT_WARP);
  }
  for (int32_t m = T - 1; m >= 1; --m) {                 // then TB level, one warp per TB
    const int64_t f = M.F(1, m);
    if (M.fits(f)) return done(1, m, f, CATT_FIT_CTA);
  }
  return done(W, T, full, CATT_FIT_UNRESOLVABLE);
}

extern "C" catt_status catt_hw_titanv(catt_hw* out) {
  if (!out) return CATT_EINVAL;
  std::memset(out, 0, sizeof(*out));
  out->num_sms = 80;          // Table 1
  out->max_warps_sm = 64;
  out->max_ctas_sm = 32;
  out->regs_sm = 65536;       // 256 KB register file
  out->reg_alloc_unit = 256;
  out->warp_size = 32;
  out->smem_alloc_unit = 256;
  out->reserved_smem_cta = 0;
  out->line_bytes = 128;
  const int32_t carve[6] = {0, 8, 16, 32, 64, 96};
  out->n_carveouts = 6;
  for (int i = 0; i < 6; ++i) {
    out->carveout_kb[i] = carve[i];
    out->carveout_pct[i] = int32_t(ceil_div(int64_t(carve[i]) * 100, 96));
    out->l1d_bytes[i] = int64_t(128 - carve[i]) * 1024;   // 128 KB shared by L1D and smem
  }
  return CATT_OK;
}

extern "C" catt_status catt_hw_b200(catt_hw* out) {
  if (!out) return CATT_EINVAL;
  std::memset(out, 0, sizeof(*out));
  out->num_sms = 148;
  out->max_warps_sm = 64;
  out->max_ctas_sm = 32;
  out->regs_sm = 65536;
  out->reg_alloc_unit = 256;
  out->warp_size = 32;
  out->smem_alloc_unit = 128;
  out->reserved_smem_cta = 1024;   // cudaDevAttrReservedSharedMemoryPerBlock
  out->line_bytes = 128;
  // B200 rule (readings R18, R19): a request must touch >= 8 lines for its
  // misses to cost more than the TLP a throttle gives up (ncu study,
  // profiles/round1_ncu_cases_a_raw.csv); at least 8 active warps per SM (2 per
  // sub-partition), calibrated on the swept launches of profiles/r1/.
  out->min_warps_sm = 8;
  out->divergent_lines = 8;
  // R23 (round 1, after the final pass): a throttle must be paid for by
  // enough reuse: a thread re-touches its line >= 16 times (VEC4's 16-byte
  // steps give 8: full TLP measured 1.23x faster than the guarded pick).
  // R23's reuse-trip term (>= 128 iterations) is off since R24: held-out
  // study 2 (profiles/r1q/) showed short scalar rows (96 iterations) gain
  // 1.3x from a throttle while the KM transpose loses at every trip count
  // (16 .. 256); what sets the transpose apart is its store stream (R24).
  out->min_retouch = 16;
  out->min_reuse_trip = 0;
  out->max_stream_pct = 25;
  // R27 (after held-out set 7, restricted to T >= 2): the floor fallback caps
  // whole CTAs when an SM holds several
  out->cta_fallback = 1;
  // R29 (round 2, held-out study 10, picks pre-registered): with one CTA per
  // SM, S >= 2 divergent streams lower the TLP floor to ceil(8 / S):
  // 14/18 launches within 5 % of the best (7/18 without), geomean 1.019x
  // (1.106x), worst 1.076x (1.373x) (profiles/r2/heldout10/)
  out->stream_floor = 1;
  // R32 (round 2, held-out study 11, picks pre-registered): a divergent load
  // whose lines every warp of the CTA shares (SYRK/SYR2K's a[j][k]) is not a
  // stream: 14/17 launches within 5 % of the best (10/17 without), geomean
  // 1.016x (1.089x), worst 1.089x (1.359x) (profiles/r2/heldout11/)
  out->private_streams = 1;
  // Shared-memory options (KB) and the carveout percentage that selects each
  // (percent of the 228 KB maximum; the driver rounds up to the next option).
  // L1D capacity per option, measured on B200 by the Fig 3-style sweep
  // (profiles/round1_probe_hw.txt): the largest cyclic footprint still served
  // from L1 is about 250 KB - option for options >= 64 KB, and 218 KB for every
  // percentage that maps to an option <= 32 KB.
  const int32_t carve[10] = {0, 8, 16, 32, 64, 100, 132, 164, 196, 228};
  const int32_t pct[10] = {0, 1, 4, 8, 15, 29, 44, 58, 72, 86};
  const int32_t l1d_kb[10] = {218, 218, 218, 218, 186, 150, 118, 86, 53, 21};
  out->n_carveouts = 10;
  for (int i = 0; i < 10; ++i) {
    out->carveout_kb[i] = carve[i];
    out->carveout_pct[i] = pct[i];
    out->l1d_bytes[i] = int64_t(l1d_kb[i]) * 1024;
  }
  return CATT_OK;
}
