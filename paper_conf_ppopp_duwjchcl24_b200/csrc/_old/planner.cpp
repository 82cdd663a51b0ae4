// Algorithm 1 planner + the host-only planner C-ABI used by the CPU tests.
#include "planner.h"

#include <stdint.h>
#include <string.h>

#include <deque>
#include <memory>
#include <vector>

#include "../../include/liger.h"

namespace liger {

void plan_round(const std::vector<Cursor*>& plist, double cf, RoundPlan* out) {
  out->sub0.clear();
  out->sub1.clear();
  out->time0 = out->time1_scaled = 0;
  if (plist.empty()) return;
  Cursor* prim = plist[0];
  double time = 0;
  int type = KT_COMPUTE;
  // (2) primary subset up to and including the switch point
  while (!prim->empty()) {
    const int left = prim->head_left();
    type = prim->head_type();
    time += prim->head_dur(left);
    const int nt = prim->next_type();
    out->sub0.push_back(PlannedPiece{0, prim->take(left), left, false});
    if (nt < 0 || nt != type) break;
  }
  out->type = type;
  out->time0 = time;
  // (3) subsequent batches fill the window with kernels of the other type
  for (size_t v = 1; v < plist.size() && time > 0; ++v) {
    Cursor* V = plist[v];
    while (time > 0 && !V->empty() && V->head_type() != type) {
      const int left = V->head_left();
      const double c = cf * V->head_dur(left);
      if (c <= time) {
        out->sub1.push_back(PlannedPiece{(int)v, V->take(left), left, false});
        time -= c;
        out->time1_scaled += c;
      } else if (V->head_decomposable() && left > 1) {
        int best = 0;
        for (int k = 1; k < left; ++k)
          if (cf * V->head_dur(k) <= time) best = k;
        if (best == 0) {
          time = 0;
        } else {
          const double cb = cf * V->head_dur(best);
          out->sub1.push_back(PlannedPiece{(int)v, V->take(best), best, true});
          time -= cb;
          out->time1_scaled += cb;
        }
      } else {
        time = 0;
      }
    }
  }
}

// ------------------------------------------------------------------ explicit-list cursor (tests)
struct ListKernel {
  int type, units, done;
  std::vector<double> durs;   // durs[k-1] = duration of k units
};

struct ListCursor : Cursor {
  int64_t batch;
  std::deque<ListKernel> ks;
  int64_t next_index = 0;     // index of ks.front() in the original list
  bool empty() const override { return ks.empty(); }
  int head_type() const override { return ks.front().type; }
  int head_left() const override { return ks.front().units - ks.front().done; }
  bool head_decomposable() const override { return ks.front().units > 1; }
  double head_dur(int k) const override { return ks.front().durs[k - 1]; }
  int next_type() const override { return ks.size() > 1 ? ks[1].type : -1; }
  int64_t take(int k) override {
    ListKernel& h = ks.front();
    const int u0 = h.done;
    h.done += k;
    // token: kernel index (high bits) | u0 (bits 8..15) | u1 (bits 0..7)
    const int64_t tok = (next_index << 16) | ((int64_t)u0 << 8) | (int64_t)h.done;
    if (h.done == h.units) {
      ks.pop_front();
      ++next_index;
    }
    return tok;
  }
};

}  // namespace liger

struct liger_planner {
  int list_size;
  double cf;
  std::deque<std::unique_ptr<liger::ListCursor>> waiting;
  std::vector<std::unique_ptr<liger::ListCursor>> processing;
};

using namespace liger;

extern "C" {

int liger_planner_create(int list_size, double cf, liger_planner** out) {
  if (!out || list_size < 1) return LIGER_EINVAL;
  *out = new liger_planner{list_size, cf > 0 ? cf : 1.0, {}, {}};
  return LIGER_OK;
}

int liger_planner_submit(liger_planner* p, int64_t batch, int n_kernels, const int32_t* types, const int32_t* units,
                         const double* durs) {
  if (!p || n_kernels < 0) return LIGER_EINVAL;
  auto c = std::make_unique<ListCursor>();
  c->batch = batch;
  size_t off = 0;
  for (int i = 0; i < n_kernels; ++i) {
    ListKernel k{types[i], units[i], 0, {}};
    if (k.units < 1 || k.units > 255) return LIGER_EINVAL;
    k.durs.assign(durs + off, durs + off + k.units);
    off += k.units;
    c->ks.push_back(std::move(k));
  }
  p->waiting.push_back(std::move(c));
  return LIGER_OK;
}

// entries: [cap][5] = {batch, kernel index, unit begin, unit end, subset}
int liger_plan_round(liger_planner* p, int32_t* entries, int cap, int32_t* n_out, int32_t* round_type,
                     double* time0) {
  if (!p) return LIGER_EINVAL;
  if (n_out) *n_out = 0;
  // update_list(): drop exhausted batches, admit FIFO from the waiting queue
  std::vector<std::unique_ptr<ListCursor>> keep;
  for (auto& c : p->processing)
    if (!c->empty()) keep.push_back(std::move(c));
  p->processing.swap(keep);
  while ((int)p->processing.size() < p->list_size && !p->waiting.empty()) {
    p->processing.push_back(std::move(p->waiting.front()));
    p->waiting.pop_front();
  }
  if (p->processing.empty()) return LIGER_IDLE;
  std::vector<Cursor*> pl;
  for (auto& c : p->processing) pl.push_back(c.get());
  RoundPlan r;
  plan_round(pl, p->cf, &r);
  int n = 0;
  auto emit = [&](const PlannedPiece& pp, int subset) {
    if (n < cap) {
      int32_t* e = entries + 5 * n;
      e[0] = (int32_t)p->processing[pp.cursor]->batch;
      e[1] = (int32_t)(pp.token >> 16);
      e[2] = (int32_t)((pp.token >> 8) & 0xff);
      e[3] = (int32_t)(pp.token & 0xff);
      e[4] = subset;
    }
    ++n;
  };
  for (auto& pp : r.sub0) emit(pp, 0);
  for (auto& pp : r.sub1) emit(pp, 1);
  if (round_type) *round_type = r.type;
  if (time0) *time0 = r.time0;
  if (n_out) *n_out = n;
  return n <= cap ? LIGER_OK : LIGER_EINVAL;
}

int liger_planner_destroy(liger_planner* p) {
  delete p;
  return LIGER_OK;
}

}  // extern "C"
