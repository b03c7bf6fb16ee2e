// plan.h — the launch geometry of one AllReduce call (host, pure functions).
//
// Every CTA of the tree kernel spins on CTAs of other ranks, and the two ends of an
// edge must cut every chunk into the SAME J channel slices (a per-channel counter
// describes one byte range on both sides, a3).  So J must be a function of
// quantities every rank knows identically — the trees, the process layout, the
// agreed settings and the buffer size — never of one process's own task count.
// These functions compute it for any process of the communicator; the runtime uses
// them with the maximum over all processes, and ccube_plan_launch exposes them to
// the host-only tests.
#pragma once
#include <stdint.h>

#include "trees.h"

namespace ccube {

struct PlanIn {
  const Tree *trees;   // [ntrees]
  int ntrees;
  int world;           // P
  int nlocal;          // ranks per process (1, or P in loopback)
  int transport;       // CCUBE_TRANSPORT_*
  int overlap;         // 1 = C1, 0 = B
  bool sgd;            // fused SGD update (adds an UPDATE task per leaf and channel)
  uint64_t bytes;      // buffer bytes of this call
  uint64_t chunk_bytes;
  bool split_heads;    // the pipeline's head tasks run on two CTAs per channel
};

// The pipeline's head: an UP task whose children are all pulled leaves (it reads its
// own and its children's inputs from DRAM).  Split over two CTAs per channel when
// PlanIn::split_heads.
bool plan_is_head(const PlanIn &in, const Tree &tr, int r);

// Edge child -> parent: PULL (the parent reads the child's partial in place) when
// both ranks live in the same process (same GPU) under AUTO; PUSH otherwise.
bool plan_edge_is_pull(int transport, int nlocal, int child, int parent);

// CTAs process `proc` launches with J channels (the task table of runtime.cc): J
// per UP / DOWN / UPDATE task, plus ONE leaf-group CTA per rank for all the trees in
// which it is a pulled leaf (a pulled leaf only publishes its heads and waits for its
// result).
int plan_tasks_of_proc(const PlanIn &in, int proc, int J);

// Maximum over every process of the communicator.
int plan_max_tasks(const PlanIn &in, int J);

// Auto channel count: the most channels whose CTAs fit `cap` co-resident CTAs on
// EVERY process (max over processes), capped at one channel per two 2 KB units of
// a chunk while the buffer is shorter than 16 chunks, one per unit beyond.
int plan_auto_channels(const PlanIn &in, int cap);

}  // namespace ccube
