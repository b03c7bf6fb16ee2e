// trees.cc — a1, the logical tree(s) of the library (host, pure).
//
// Paper: the pipelined tree of Fig 5(a), root N4 <- N2 <- {N1, N3}, and
// the double binary tree whose second tree is the first "flipped to invert the
// nodes and leaves" (fn4 P:L153).  Reading R1: binary tree
// rooted at rank 0 with one child; rank r (lowest set bit b) has children
// r - b/2 and r + b/2, the right offset halved until it is < P.  Tree 1 renames
// every rank v of tree 0 to P-1-v (even P) or (v+1) mod P (odd P).  The ROTATED
// set renames tree 0 by v -> (v + t) mod P for t = 0..P-1.
//
// This builder works top-down from the children rule; the oracle builds the same
// tree bottom-up from a parent rule, and tests/test_abi_host.py checks that the
// two agree for every P.
#include "trees.h"

#include <algorithm>
#include <limits>

namespace ccube {

namespace {

void build_tree0(int P, Tree *t) {
  t->P = P;
  t->root = 0;
  for (int v = 0; v < P; ++v) {
    t->parent[v] = -1;
    t->nchild[v] = 0;
  }
  if (P <= 1) return;
  int top = 1;
  while (top * 2 < P) top *= 2;  // largest power of two below P
  t->nchild[0] = 1;
  t->child[0][0] = top;
  t->parent[top] = 0;
  // breadth-first over the power-of-two offsets
  for (int b = top; b >= 2; b /= 2) {
    for (int r = b; r < P; r += 2 * b) {
      if ((r & -r) != b) continue;
      const int left = r - b / 2;
      t->child[r][t->nchild[r]++] = left;
      t->parent[left] = r;
      int off = b / 2;
      while (off > 0 && r + off >= P) off /= 2;
      if (off > 0) {
        t->child[r][t->nchild[r]++] = r + off;
        t->parent[r + off] = r;
      }
    }
  }
}

int rename(int P, int kind, int which, int v) {
  if (kind == 2) return (v + which) % P;
  return (P % 2 == 0) ? (P - 1 - v) : ((v + 1) % P);
}

}  // namespace

int num_trees(int P, int kind) { return kind == 2 ? (P > 1 ? P : 1) : kind == 1 ? 2 : 1; }

void build_tree(int P, int kind, int which, Tree *out) {
  Tree t0;
  build_tree0(P, &t0);
  if (which == 0) {
    *out = t0;
    return;
  }
  out->P = P;
  out->root = rename(P, kind, which, t0.root);
  for (int v = 0; v < P; ++v) out->nchild[v] = 0;
  for (int v = 0; v < P; ++v) {
    const int nv = rename(P, kind, which, v);
    out->parent[nv] = t0.parent[v] < 0 ? -1 : rename(P, kind, which, t0.parent[v]);
  }
  // children in ascending rank (the combine order, R2)
  for (int c = 0; c < P; ++c) {
    const int p = out->parent[c];
    if (p >= 0) out->child[p][out->nchild[p]++] = c;
  }
}

void place_tree(const int *perm, Tree *t) {
  const int P = t->P;
  int parent[kTreeMaxP];
  for (int v = 0; v < P; ++v)
    parent[perm[v]] = t->parent[v] < 0 ? -1 : perm[t->parent[v]];
  for (int v = 0; v < P; ++v) {
    t->parent[v] = parent[v];
    t->nchild[v] = 0;
    if (parent[v] < 0) t->root = v;
  }
  for (int c = 0; c < P; ++c)  // ascending rank
    if (parent[c] >= 0) t->child[parent[c]][t->nchild[parent[c]]++] = c;
}

bool plan_placement(int P, int kind, const double *bw, int *perm) {
  if (P < 1 || P > 8) return false;
  // directed edge loads of the identity placement, in units of 1/T of the buffer
  int load[8][8] = {};
  const int T = num_trees(P, kind);
  for (int t = 0; t < T; ++t) {
    Tree tr;
    build_tree(P, kind, t, &tr);
    for (int c = 0; c < P; ++c) {
      if (tr.parent[c] < 0) continue;
      ++load[c][tr.parent[c]];
      ++load[tr.parent[c]][c];
    }
  }
  int p[8];
  for (int v = 0; v < P; ++v) p[v] = perm[v] = v;
  double best = std::numeric_limits<double>::infinity();
  bool first = true;
  do {  // lexicographic order from the identity; strict improvement only
    double cost = 0.0;
    for (int i = 0; i < P; ++i)
      for (int j = 0; j < P; ++j) {
        if (!load[i][j]) continue;
        const double b = bw[p[i] * P + p[j]];
        const double c = b > 0 ? (static_cast<double>(load[i][j]) / T) / b
                               : std::numeric_limits<double>::infinity();
        cost = std::max(cost, c);
      }
    if (first || cost < best) {
      best = cost;
      first = false;
      for (int v = 0; v < P; ++v) perm[v] = p[v];
    }
  } while (std::next_permutation(p, p + P));
  return true;
}

int child_slot(const Tree &t, int parent, int c) {
  for (int s = 0; s < t.nchild[parent]; ++s)
    if (t.child[parent][s] == c) return s;
  return -1;
}

}  // namespace ccube
