// set-associative LRU simulation of sector (32 B) accesses: returns misses
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
int64_t simulate(const int32_t* cols, int64_t n, int64_t sets, int ways, int elem_bytes, int64_t warm) {
    int64_t* tag = (int64_t*)malloc(sizeof(int64_t) * sets * ways);
    uint32_t* age = (uint32_t*)calloc(sets * ways, sizeof(uint32_t));
    for (int64_t i = 0; i < sets * ways; ++i) tag[i] = -1;
    uint32_t clock = 0;
    int64_t miss = 0;
    for (int pass = 0; pass < 2; ++pass) {          // pass 0 warms the cache (steady state across steps)
        for (int64_t i = 0; i < n; ++i) {
            int32_t c = cols[i];
            if (c < 0) continue;
            int64_t sec = ((int64_t)c * elem_bytes) >> 5;
            uint64_t h = (uint64_t)sec * 0x9E3779B97F4A7C15ull;
            int64_t s = (int64_t)((h >> 20) % (uint64_t)sets);
            int64_t* t = tag + s * ways;
            uint32_t* a = age + s * ways;
            ++clock;
            int hit = -1, lru = 0;
            for (int w = 0; w < ways; ++w) {
                if (t[w] == sec) { hit = w; break; }
                if (a[w] < a[lru]) lru = w;
            }
            if (hit >= 0) a[hit] = clock;
            else { if (pass == 1) ++miss; t[lru] = sec; a[lru] = clock; }
        }
    }
    free(tag); free(age);
    return miss;
}
