// Host-only check of the host-mapped decision record protocol (MappedRec,
// common.cuh): the device writes four 16-byte chunks, each three payload
// words and a tag = seq ^ mix(payload, chunk), with no fence; the host
// accepts the record only when all four tags match the sequence number it
// waits for. Chunks are written here exactly as publish_mapped writes them
// (rec_payload + rec_tag), then stale, torn and corrupted states are read.
#include <cmath>
#include <cstdio>

#include "../../paper_conf_sc_cui0czlzsmylg21_b200/csrc/common.cuh"

using namespace abacus;

static void write_chunk(MappedRec& M, const Result& R, uint32_t seq, int i) {
    uint32_t p[12];
    rec_payload(R, p);
    M.w[4 * i] = p[3 * i];
    M.w[4 * i + 1] = p[3 * i + 1];
    M.w[4 * i + 2] = p[3 * i + 2];
    M.w[4 * i + 3] = rec_tag(seq, p[3 * i], p[3 * i + 1], p[3 * i + 2], (uint32_t)i);
}
static void publish(MappedRec& M, const Result& R, uint32_t seq) {
    for (int i = 0; i < 4; i++) write_chunk(M, R, seq, i);
}
static Result sample(uint32_t s) {
    Result R{};
    R.key = (0x123ull + s) << 40 | (0xABCDEull * s);
    R.y_best = 15.25f + (float)s;
    R.y0 = 40.5f - (float)s;
    R.evaluated = 9188218208ull + s;
    for (int j = 0; j < kKMax; j++) R.end_op[j] = (int32_t)(100 * j + s);
    R.total_ops = 1205 + (int32_t)s;
    R.status = (int32_t)(s % 3);
    R.pad = 77 + s;
    return R;
}
static bool same(const Result& a, const Result& b) {
    if (a.key != b.key || a.evaluated != b.evaluated || a.total_ops != b.total_ops || a.status != b.status ||
        a.pad != b.pad || memcmp(&a.y_best, &b.y_best, 4) || memcmp(&a.y0, &b.y0, 4))
        return false;
    for (int j = 0; j < kKMax; j++)
        if (a.end_op[j] != b.end_op[j]) return false;
    return true;
}

int main() {
    int bad = 0;
#define CHECK(c)                                               \
    do {                                                       \
        if (!(c)) {                                            \
            fprintf(stderr, "FAIL line %d: %s\n", __LINE__, #c); \
            bad++;                                             \
        }                                                      \
    } while (0)
    MappedRec M{};
    Result R{};
    // zeroed memory (a fresh context) matches no sequence number
    for (uint32_t s = 1; s < 2000; s++) CHECK(!rec_read(&M, s, &R));
    // a complete record is accepted for its own number only, and read back exactly
    const Result A = sample(7);
    publish(M, A, 7);
    CHECK(rec_read(&M, 7, &R) && same(R, A));
    CHECK(!rec_read(&M, 8, &R));
    // NaN payloads survive the round trip bit for bit
    Result N = sample(9);
    N.y_best = NAN;
    publish(M, N, 9);
    CHECK(rec_read(&M, 9, &R) && std::isnan(R.y_best) && R.key == N.key);
    // the next decision's record arriving chunk by chunk: stale until the last chunk lands
    publish(M, A, 7);
    const Result B = sample(8);
    for (int i = 0; i < 4; i++) {
        CHECK(!rec_read(&M, 8, &R));
        write_chunk(M, B, 8, i);
    }
    CHECK(rec_read(&M, 8, &R) && same(R, B));
    CHECK(!rec_read(&M, 7, &R));
    // a torn 16-byte chunk (payload of the new record, tag of the old) is refused
    for (int i = 0; i < 4; i++) {
        publish(M, B, 8);
        uint32_t p[12];
        rec_payload(sample(10), p);
        M.w[4 * i] = p[3 * i];  // one payload word from record 10, the rest from 8
        CHECK(!rec_read(&M, 8, &R));
        CHECK(!rec_read(&M, 10, &R));
    }
    // single-bit corruption of any word is refused
    for (int wd = 0; wd < 16; wd++)
        for (int bit = 0; bit < 32; bit += 7) {
            publish(M, B, 8);
            M.w[wd] ^= 1u << bit;
            CHECK(!rec_read(&M, 8, &R));
        }
    if (bad) return 1;
    printf("mapped record protocol: ok\n");
    return 0;
}
