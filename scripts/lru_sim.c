/* Fully associative LRU simulation of a row-gather stream (analysis only).
 * lru_misses(n, stream, len, cap) -> number of misses when `stream` (row ids
 * in [0,n)) is gathered through an LRU cache holding `cap` rows.
 * Build: gcc -O2 -shared -fPIC -o scripts/liblrusim.so scripts/lru_sim.c */
#include <stdint.h>
#include <stdlib.h>

int64_t lru_misses(int64_t n, const int32_t *s, int64_t len, int64_t cap) {
  int32_t *prv = malloc(sizeof(int32_t) * n), *nxt = malloc(sizeof(int32_t) * n);
  uint8_t *in = calloc(n, 1);
  int32_t head = -1, tail = -1;
  int64_t size = 0, miss = 0;
  for (int64_t k = 0; k < len; ++k) {
    int32_t v = s[k];
    if (in[v]) {
      if (head == v) continue;
      /* unlink */
      nxt[prv[v]] = nxt[v];
      if (nxt[v] >= 0) prv[nxt[v]] = prv[v]; else tail = prv[v];
    } else {
      ++miss;
      in[v] = 1;
      if (++size > cap) {
        int32_t t = tail;
        tail = prv[t];
        nxt[tail] = -1;
        in[t] = 0;
        --size;
      }
    }
    prv[v] = -1;
    nxt[v] = head;
    if (head >= 0) prv[head] = v;
    head = v;
    if (tail < 0) tail = v;
  }
  free(prv); free(nxt); free(in);
  return miss;
}
