// tile_check.cpp -- CPU check of the segment-table tile layout: the host
// layout (tables.h:seg_layout, what the executor writes into each SegDesc) and the
// element ranges the kernels derive from it (tables.h:tile_range, the same function the
// sm_100a kernels call) partition [0, n) of every VP exactly -- no gap, no overlap, no
// padding -- and every tile on the vector path starts 16-B aligned and is whole.
// Built and run by tests/test_tiles.py; prints "OK <cases>" or the first failing case.
#include <stdio.h>

#include <random>
#include <vector>

#include "../paper_conf_dac_jungc15_b200/csrc/tables.h"

using namespace svp;

static int check(uint64_t ptr0, bool co, int es, int T, uint64_t n) {
    uint16_t shift;
    uint64_t nt;
    bool scalar;
    seg_layout(ptr0, co, es, T, n, &shift, &nt, &scalar);
    const uint32_t flags = scalar ? SEG_SCALAR : 0;
    int64_t prev = 0;
    int nonvec = 0;
    for (uint64_t lt = 0; lt < nt; ++lt) {
        int64_t e0, e1;
        bool vec;
        tile_range(n, shift, flags, (uint32_t)lt, T, e0, e1, vec);
        if (e0 != prev || e1 <= e0) return 1;                           // contiguous, non-empty
        if (vec && (e1 - e0 != T || (ptr0 + (uint64_t)e0 * es) % 16 != 0)) return 2;  // aligned, whole
        if (vec && scalar) return 3;
        if (!vec) ++nonvec;
        prev = e1;
    }
    if ((uint64_t)prev != n) return 4;                                 // covers [0, n) exactly
    if (!scalar && nonvec > 2) return 5;                               // only head / tail tiles
    if (!scalar && co && (ptr0 % 16) % es == 0 && shift != (ptr0 % 16) / es) return 6;
    return 0;
}

int main() {
    std::mt19937_64 g(12345);
    long cases = 0;
    const int tiles[] = {kVecaddTile, kBsTile, kHistTile};
    for (int T : tiles) {
        for (int es : {1, 4}) {
            for (int mis = 0; mis < 16; ++mis) {
                for (int co = 0; co < 2; ++co) {
                    std::vector<uint64_t> ns = {0, 1, 2, 3, 4, 5, 15, 16, 17, (uint64_t)T - 1, (uint64_t)T,
                                                (uint64_t)T + 1, 2ull * T - 1, 2ull * T + 3, 5ull * T + 7};
                    for (int r = 0; r < 200; ++r) ns.push_back(g() % (uint64_t)(40 * T));
                    for (uint64_t n : ns) {
                        const uint64_t ptr0 = 0x7f0000000000ull + 256ull * (g() % 4096) + (uint64_t)mis;
                        const int rc = check(ptr0, co != 0, es, T, n);
                        ++cases;
                        if (rc) {
                            printf("FAIL rc=%d T=%d es=%d mis=%d co=%d n=%llu\n", rc, T, es, mis, co,
                                   (unsigned long long)n);
                            return 1;
                        }
                    }
                }
            }
        }
    }
    printf("OK %ld\n", cases);
    return 0;
}
