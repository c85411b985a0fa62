/* tools/lru_model.c -- L2-capacity model for B-row reuse (SURVEY.md §8(d) "Ceiling note").
 * Replays the B-row accesses of an SpMM in a given row order (rows in `order`, each row's columns in
 * CSR order) through a fully-associative LRU cache of `cap` B rows and counts misses.  Measurement
 * helper only (not part of the method, not part of the oracle). */
#include <stdint.h>
#include <stdlib.h>

int64_t lru_misses(int64_t M, int64_t N, const int64_t *rowidx, const int32_t *colidx, const int32_t *order,
                   int64_t cap) {
    int32_t *prev = (int32_t *)malloc(N * sizeof(int32_t)), *next = (int32_t *)malloc(N * sizeof(int32_t));
    char *in = (char *)calloc(N, 1);
    int32_t head = -1, tail = -1;   /* head = most recent */
    int64_t size = 0, misses = 0;
    for (int64_t p = 0; p < M; ++p) {
        int64_t i = order ? order[p] : p;
        for (int64_t j = rowidx[i]; j < rowidx[i + 1]; ++j) {
            int32_t c = colidx[j];
            if (in[c]) {
                if (c == head) continue;
                /* unlink */
                if (prev[c] >= 0) next[prev[c]] = next[c];
                if (next[c] >= 0) prev[next[c]] = prev[c];
                if (tail == c) tail = prev[c];
            } else {
                ++misses;
                if (size == cap) {   /* evict tail */
                    int32_t t = tail;
                    tail = prev[t];
                    if (tail >= 0) next[tail] = -1;
                    in[t] = 0;
                    --size;
                    if (head == t) head = -1;
                }
                in[c] = 1;
                ++size;
            }
            prev[c] = -1;
            next[c] = head;
            if (head >= 0) prev[head] = c;
            head = c;
            if (tail < 0) tail = c;
        }
    }
    free(prev); free(next); free(in);
    return misses;
}
