// trees.h — logical tree tables (a1).  See trees.cc.
#pragma once

namespace ccube {

constexpr int kTreeMaxP = 64;

struct Tree {
  int P;
  int root;
  int parent[kTreeMaxP];      // -1 at the root
  int nchild[kTreeMaxP];      // 0..2
  int child[kTreeMaxP][2];    // ascending rank
};

// Tree kinds (ccube_tree_kind_t): 0 single, 1 double, 2 rotated.
int num_trees(int P, int kind);
// Tree `which` of `kind`: which = 0 is the first tree (root 0); DOUBLE's tree 1 is
// the flipped tree; ROTATED's tree t is tree 0 with ranks renamed (v + t) mod P.
void build_tree(int P, int kind, int which, Tree *out);

// Position of c among parent's children (the receive plane it writes), -1 if none.
int child_slot(const Tree &t, int parent, int c);

// Placement (reading R19, the NVSwitch form of §IV's detours): tree
// position v is hosted by rank perm[v]; children are re-listed in ascending rank
// (the combine order, R2).  perm must be a permutation of 0..P-1.
void place_tree(const int *perm, Tree *t);

// The least-cost placement for a measured P x P peer bandwidth matrix bw[i*P + j]
// (i -> j, any unit): every tree carries 1/T of the buffer up and down each of its
// edges, and the cost of a placement is max over loaded directed pairs of
// load / bw.  Exhaustive over the P! placements (P <= 8), ties to the
// lexicographically smallest, so uniform bandwidth keeps the identity.
// Returns false for P > 8.
bool plan_placement(int P, int kind, const double *bw, int *perm);

}  // namespace ccube
