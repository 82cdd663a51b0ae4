// Algorithm 1 (§3.4) with the contention factor (§3.5,
// P:248) and runtime decomposition (§3.6).  Pure host code.
//
// Readings: R1 the printed comparator is inverted -- a secondary
// kernel is taken when cf*dur <= remaining time; R2 the end of the primary's
// list counts as a switch point; R3 cf multiplies every secondary duration;
// R5 a secondary kernel that does not fit is decomposed into the largest k/F
// piece that fits, the remainder stays at the head of its batch.
#pragma once
#include <stdint.h>

#include <vector>

namespace liger {

enum KType { KT_COMPUTE = 0, KT_COMM = 1 };

// A batch's kernel list as seen by the planner ("function wrappers", §3.2).
struct Cursor {
  virtual ~Cursor() {}
  virtual bool empty() const = 0;
  virtual int head_type() const = 0;
  virtual int head_left() const = 0;            // units not yet launched (1 if not decomposable)
  virtual bool head_decomposable() const = 0;
  virtual double head_dur(int k) const = 0;     // profiled duration of k more units of the head
  virtual int next_type() const = 0;            // type of the kernel after the head, -1 if none
  // Remove k units of the head kernel; returns an opaque token describing the piece.
  virtual int64_t take(int k) = 0;
};

struct PlannedPiece {
  int cursor;      // index in the processing list
  int64_t token;   // from Cursor::take
  int units;       // units in this piece
  bool partial;    // k < the kernel's remaining units
};

struct RoundPlan {
  std::vector<PlannedPiece> sub0, sub1;
  int type = KT_COMPUTE;
  double time0 = 0, time1_scaled = 0;
};

// One iteration of Algorithm 1 over the processing list (index 0 = primary).
void plan_round(const std::vector<Cursor*>& plist, double cf, RoundPlan* out);

}  // namespace liger
