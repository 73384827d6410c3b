// Host test of raw_threshold (device_common.cuh): y_raw <= T decides exactly
// what fl(y_raw + b4) <= H decides, for random and edge-case (H, b4, y_raw),
// compiled with nvcc against the library's own header.
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <random>

#include "../../paper_conf_sc_cui0czlzsmylg21_b200/csrc/device_common.cuh"

using abacus::add_rn;
using abacus::raw_threshold;

static int fails = 0;
static void check(float H, float b4, float yr) {
    const float T = raw_threshold(H, b4);
    const bool a = add_rn(yr, b4) <= H, b = yr <= T;
    if (a != b) {
        if (fails++ < 10) printf("mismatch H=%a b4=%a yr=%a T=%a\n", H, b4, yr, T);
    }
}

int main() {
    std::mt19937_64 rng(20261018);
    std::uniform_real_distribution<float> uH(0.5f, 200.0f), ub(-5.0f, 50.0f);
    for (int i = 0; i < 20000; i++) {
        const float H = uH(rng), b4 = ub(rng);
        const float T = raw_threshold(H, b4);
        // T is the largest raw value that fits
        if (!(add_rn(T, b4) <= H) || add_rn(nextafterf(T, INFINITY), b4) <= H) {
            if (fails++ < 10) printf("not maximal H=%a b4=%a T=%a\n", H, b4, T);
        }
        // raw values around the threshold and random ones
        float y = T;
        for (int k = 0; k < 8; k++) y = nextafterf(y, -INFINITY);
        for (int k = 0; k < 16; k++, y = nextafterf(y, INFINITY)) check(H, b4, y);
        std::uniform_real_distribution<float> uy(H - b4 - 1.0f, H - b4 + 1.0f);
        for (int k = 0; k < 16; k++) check(H, b4, uy(rng));
    }
    // edge cases: exact ties, b4 = 0, large b4, H = +inf / NaN
    const float Hs[] = {1.0f, 33.486f, 1e-3f, 1e6f, INFINITY, NAN};
    const float bs[] = {0.0f, 2.0f, -2.0f, 1e5f, 3.0e-8f};
    for (float H : Hs)
        for (float b4 : bs)
            for (float yr : {0.0f, 1.0f, -1.0f, 33.486f - 2.0f, 31.486f, 1e6f, -1e6f, INFINITY, -INFINITY})
                check(H, b4, yr);
    if (fails) {
        printf("%d failures\n", fails);
        return 1;
    }
    printf("ok\n");
    return 0;
}
