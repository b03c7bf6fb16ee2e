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

// which = 0: first tree (root 0); which = 1: the flipped second tree.
void build_tree(int P, int which, Tree *out);

// Position of c among parent's children (the receive plane it writes), -1 if none.
int child_slot(const Tree &t, int parent, int c);

}  // namespace ccube
