// Host check that the replay kernel's raw-flag label + expanded table (label_raw,
// expand_raw_table in include/hirace_device.cuh) select exactly the canonical FSM entry
// (label + the 2048-entry table of PAPER.md L295's flat-array encoding) for every state, kind,
// thread relation and epoch difference, in power-of-two and general geometries.
// Usage: label_raw_check <table.bin>   (2048 bytes from hirace_fsm_table); exit 0 = equal.
#include <cstdio>
#include <cstdlib>
#include <random>

#include "hirace_device.cuh"

using namespace hirace;

int main(int argc, char **argv)
{
    if (argc < 2)
        return 2;
    unsigned char canon[2048], raw[RAW_TABLE_BYTES];
    FILE *f = std::fopen(argv[1], "rb");
    if (!f || std::fread(canon, 1, 2048, f) != 2048)
        return 2;
    std::fclose(f);
    expand_raw_table(canon, raw);
    const uint32_t geoms[][2] = {{256, 32}, {64, 32}, {32, 64}, {8, 2}, {6, 2}, {96, 32}, {1, 1}, {1024, 32}};
    std::mt19937_64 rng(20241117);
    long checked = 0;
    for (auto &gm : geoms) {
        hirace_dev_ctx c{};
        c.block_threads = gm[0];
        c.warp_size = gm[1];
        fastdiv_init(c.block_threads, &c.bt_magic, &c.bt_s1, &c.bt_s2);
        fastdiv_init(c.warp_size, &c.ws_magic, &c.ws_s1, &c.ws_s2);
        geom G = make_geom(c);
        const uint32_t nthr = 4 * gm[0];
        for (int it = 0; it < 400000; it++) {
            const uint32_t st = rng() % 23;
            const uint32_t otid = rng() % nthr, tid = (rng() & 1) ? otid : (uint32_t)(rng() % nthr);
            const uint32_t og = rng() % 3, ob = rng() % 3, ow = rng() % 3;
            access a{tid, (uint32_t)(rng() % 4), (uint32_t)(rng() % 3), (uint32_t)(rng() % 3), (uint32_t)(rng() % 3)};
            if (rng() & 1) { a.g = og; if (rng() & 1) { a.b = ob; if (rng() & 1) a.w = ow; } }
            const uint64_t o = pack(st, og, ob, ow, otid);
            const uint32_t e1 = canon[(st << 6) | label(o, a, G)];
            const uint32_t e2 = raw[(st << 7) | label_raw(o, a, G)];
            if (e1 != e2) {
                std::printf("mismatch bt=%u ws=%u st=%u otid=%u tid=%u o=(%u,%u,%u) a=(%u,%u,%u) k=%u: %u vs %u\n", gm[0],
                            gm[1], st, otid, tid, og, ob, ow, a.g, a.b, a.w, a.kind, e1, e2);
                return 1;
            }
            checked++;
        }
    }
    std::printf("ok %ld\n", checked);
    return 0;
}
