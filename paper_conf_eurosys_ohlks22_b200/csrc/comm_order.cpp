// Issue order of the partitioned gradient all-reduces on the comm stream
// (§5.1, Fig. 4(b): prioritised parameter communication; SURVEY §8f
// NEXT-4).  Pure host C++; readings C1-C3 in DESIGN.md.
//
// The comm stream is one FIFO channel.  Each bucket's all-reduce is
// partitioned into fixed chunks; a static issue order of the chunks is
// planned per step from the buckets' predicted ready times (the engine
// planner's dW completion estimates) and a chunk-duration model:
//   FIFO     : buckets in D's dW order, chunks in order (Fig. 4(a)/(c));
//   PRIORITY : whenever the channel frees up, the ready chunk of the bucket
//              with the lowest layer goes next; an idle channel waits for the
//              earliest ready bucket (Fig. 4(b): "the communication of
//              dW_1 - dW_4 is prioritized over dW_5").
// A misprediction only delays (the stream still waits for each bucket's
// dW counter before its first chunk); it never reorders a bucket's data.
#include <algorithm>
#include <vector>

#include "../../include/ooo.h"

extern "C" ooo_status ooo_comm_schedule(int32_t n_buckets, const double *ready, const int32_t *n_chunks,
                                        const double *dur, const int32_t *prio, const int32_t *fifo_rank,
                                        int32_t policy, int32_t *order_b, int32_t *order_c, double *done) {
  if (n_buckets < 0 || (n_buckets > 0 && (!ready || !n_chunks || !dur || !prio || !order_b || !order_c)))
    return OOO_ERR_INVALID_ARGUMENT;
  if (policy != 0 && policy != 1) return OOO_ERR_INVALID_ARGUMENT;
  const int B = n_buckets;
  std::vector<int> first(B + 1, 0);
  for (int b = 0; b < B; ++b) {
    if (n_chunks[b] < 1) return OOO_ERR_INVALID_ARGUMENT;
    first[b + 1] = first[b] + n_chunks[b];
  }
  std::vector<double> fin(B, 0.0);
  int n = 0;
  if (policy == 0) {
    std::vector<int> seq(B);
    for (int b = 0; b < B; ++b) seq[b] = b;
    if (fifo_rank)
      std::stable_sort(seq.begin(), seq.end(), [&](int x, int y) { return fifo_rank[x] < fifo_rank[y]; });
    double t = 0.0;
    for (int b : seq) {
      for (int c = 0; c < n_chunks[b]; ++c) {
        t = std::max(t, ready[b]) + dur[first[b] + c];
        order_b[n] = b;
        order_c[n++] = c;
      }
      fin[b] = t;
    }
  } else {
    std::vector<int> next(B, 0);
    int left = first[B];
    double t = 0.0;
    while (left > 0) {
      int pick = -1;
      double earliest = 0.0;
      bool any = false;
      for (int b = 0; b < B; ++b) {
        if (next[b] >= n_chunks[b]) continue;
        if (ready[b] <= t) {
          if (pick < 0 || prio[b] < prio[pick]) pick = b;   // ties: lower bucket index (scan order)
        } else if (!any || ready[b] < earliest) {
          earliest = ready[b];
          any = true;
        }
      }
      if (pick < 0) {   // channel idle until the earliest bucket is ready
        t = earliest;
        continue;
      }
      t += dur[first[pick] + next[pick]];
      order_b[n] = pick;
      order_c[n++] = next[pick]++;
      --left;
      if (next[pick] == n_chunks[pick]) fin[pick] = t;
    }
  }
  if (done)
    for (int b = 0; b < B; ++b) done[b] = fin[b];
  return OOO_OK;
}
