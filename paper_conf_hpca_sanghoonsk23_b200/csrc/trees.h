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

}  // namespace ccube
