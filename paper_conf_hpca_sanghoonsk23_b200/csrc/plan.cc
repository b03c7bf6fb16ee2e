// plan.cc — launch geometry (see plan.h).  Host only, pure.
#include "plan.h"

#include "ccube.h"

namespace ccube {

bool plan_edge_is_pull(int transport, int nlocal, int child, int parent) {
  if (transport == CCUBE_TRANSPORT_PUSH) return false;
  if (transport == CCUBE_TRANSPORT_PULL) return true;
  return child / nlocal == parent / nlocal;
}

bool plan_is_head(const PlanIn &in, const Tree &tr, int r) {
  if (tr.nchild[r] == 0) return false;
  for (int s = 0; s < tr.nchild[r]; ++s) {
    const int c = tr.child[r][s];
    if (tr.nchild[c] != 0 || !plan_edge_is_pull(in.transport, in.nlocal, c, r)) return false;
  }
  return true;
}

int plan_tasks_of_proc(const PlanIn &in, int proc, int J) {
  int n = 0;
  for (int i = 0; i < in.nlocal; ++i) {
    const int r = proc * in.nlocal + i;
    bool pulled = false;  // every pulled leaf of rank r shares one CTA
    for (int t = 0; t < in.ntrees; ++t) {
      const Tree &tr = in.trees[t];
      const bool root = tr.parent[r] < 0;
      const bool leaf = !root && tr.nchild[r] == 0;
      if (leaf && in.sgd) n += J;  // a leaf's fused SGD step (f2)
      if (leaf && plan_edge_is_pull(in.transport, in.nlocal, r, tr.parent[r])) {
        pulled = true;  // a pulled leaf: the rank's leaf-group CTA publishes every channel
        continue;
      }
      n += (in.split_heads && plan_is_head(in, tr, r)) ? 2 * J : J;  // UP
      if (tr.nchild[r] > 0 && (!root || !in.overlap)) n += J;  // DOWN
    }
    if (pulled) n += 1;
  }
  return n;
}

int plan_max_tasks(const PlanIn &in, int J) {
  const int nproc = in.world / in.nlocal;
  int m = 0;
  for (int p = 0; p < nproc; ++p) {
    const int n = plan_tasks_of_proc(in, p, J);
    if (n > m) m = n;
  }
  return m;
}

int plan_auto_channels(const PlanIn &in, int cap) {
  int J = 1;
  while (J < CCUBE_MAX_CHANNELS && plan_max_tasks(in, J + 1) <= cap) ++J;
  // a small buffer gets few channels, so few CTAs take part in the handshakes
  // (latency); a long one is bandwidth-bound and may use one 2 KB unit per channel
  const uint64_t first = in.bytes < in.chunk_bytes ? in.bytes : in.chunk_bytes;
  const uint64_t units = (first + 2047) / 2048;
  const uint64_t per = in.bytes >= 16 * in.chunk_bytes ? 1 : 2;
  const int jmax = units / per > 1 ? static_cast<int>(units / per) : 1;
  return J > jmax ? jmax : J;
}

}  // namespace ccube
