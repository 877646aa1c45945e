/*
 * fsm_table.cpp — builds HiRace's flat transition table (PAPER.md: "The HiRace FSM is
 * encoded as a flat array indexed by a concatenation of oState and the transition labels").
 *
 * The paper's full 25-state table lives in an external artifact; this build
 * derives its own exact machine from the race definition:
 * 23 states, labels = 4 kinds x 4 sync statuses (Us, Ws, Bs + Gs for a new grid epoch)
 * x 4 thread relations (S, W, B, G).  Entry = next_state:5 | keep:1 | report:1.
 *
 * Kind classes.  Inside one block atomics of either scope never conflict with each other:
 *   cls(R)=R, cls(AB)=cls(AG)=A, cls(W)=X.
 * Across blocks only grid-scope atomics are mutually atomic:
 *   clsG(R)=R, clsG(AG)=AG, clsG(AB)=clsG(W)=X.
 * join(x,y) = x if x==y else X.  compat(c,k) <=> c == cls(k) in {R,A};
 * compatG(c,k) <=> c == clsG(k) in {R,AG}.
 *
 * States (per location, within the current grid epoch):
 *   T(KT,KB,KG)  one thread in the current warp epoch; KT its kinds there, KB its warp's kinds
 *                in the current block epoch, KG its block's kinds in the grid epoch
 *   W(c,KB,KG)   >= 2 threads of one warp in the current warp epoch, all of class c
 *   B(c,KG)      >= 2 warps of one block in the current block epoch, all of class c
 *   G(c)         >= 2 blocks in the grid epoch, all of class c
 *   RACE_W/B/G   sticky; class = coarsest level in the first racing epoch (upgrades allowed
 *                while still in that epoch)
 * Rules, first match wins (record := the current accessor unless "keep"):
 *   0 RACE_*: Gs -> keep.  RACE_W & rel B & Us -> RACE_B (report).  RACE_W/B & rel G & !Gs
 *     -> RACE_G (report).  Otherwise keep.
 *   1 INIT or Gs -> T(cls k, cls k, clsG k)
 *   2 G(c): compatG(c,k) -> G(c) keep, else RACE_G
 *   3 rel G: compatG(KG,k) -> G(KG), else RACE_G
 *   4 Bs -> T(cls k, cls k, KG')
 *   5 B(c,KG): compat(c,k) -> B(c,KG') keep, else RACE_B
 *   6 rel B: compat(KB,k) -> B(KB,KG'), else RACE_B
 *   7 Ws -> T(cls k, KB', KG')
 *   8 W(c,KB,KG): compat(c,k) -> W(c,KB',KG') keep, else RACE_W
 *   9 rel W (state T): compat(KT,k) -> W(KT,KB',KG'), else RACE_W
 *  10 rel S (state T): T(join(KT,cls k), KB', KG') keep
 * with KB' = join(KB, cls k), KG' = join(KG, clsG k).
 */
#include <stdint.h>
#include <string.h>

#include "hirace.h"
#include "hirace_device.cuh"
#include "internal.h"

namespace {

enum Cl { C_R = 0, C_A = 1, C_AG = 2, C_X = 3 };

enum Group { G_INIT, G_T, G_W, G_B, G_G, G_RACE, G_NONE };

struct Desc {
    Group grp;
    int a, b, c; /* T: KT,KB,KG  W: c,KB,KG  B: c,KG  G: c */
};

const Desc kStates[hirace::ST_COUNT] = {
    {G_INIT, 0, 0, 0},
    {G_T, C_R, C_R, C_R},   {G_T, C_R, C_R, C_X},  {G_T, C_R, C_X, C_X}, {G_T, C_X, C_X, C_X},
    {G_T, C_A, C_A, C_AG},  {G_T, C_A, C_A, C_X},  {G_T, C_A, C_X, C_X},
    {G_W, C_R, C_R, C_R},   {G_W, C_R, C_R, C_X},  {G_W, C_R, C_X, C_X},
    {G_W, C_A, C_A, C_AG},  {G_W, C_A, C_A, C_X},  {G_W, C_A, C_X, C_X},
    {G_B, C_R, C_R, 0},     {G_B, C_R, C_X, 0},    {G_B, C_A, C_AG, 0},  {G_B, C_A, C_X, 0},
    {G_G, C_R, 0, 0},       {G_G, C_AG, 0, 0},
    {G_RACE, 1, 0, 0},      {G_RACE, 2, 0, 0},     {G_RACE, 3, 0, 0},
};

int cls_low(uint32_t k) { return k == HIRACE_READ ? C_R : (k == HIRACE_WRITE ? C_X : C_A); }
int cls_grid(uint32_t k) { return k == HIRACE_READ ? C_R : (k == HIRACE_ATOMIC_GRID ? C_AG : C_X); }
int join(int x, int y) { return x == y ? x : C_X; }
bool compat(int c, uint32_t k) { return (c == C_R || c == C_A) && c == cls_low(k); }
bool compatG(int c, uint32_t k) { return (c == C_R || c == C_AG) && c == cls_grid(k); }

int find(Group grp, int a, int b, int c)
{
    for (int s = 0; s < (int)hirace::ST_COUNT; s++) {
        const Desc &d = kStates[s];
        if (d.grp != grp || d.a != a)
            continue;
        if (grp == G_G || grp == G_RACE)
            return s;
        if (grp == G_B && d.b == b)
            return s;
        if ((grp == G_T || grp == G_W) && d.b == b && d.c == c)
            return s;
    }
    return -1; /* unreachable for consistent tuples; checked by the caller */
}

struct Out {
    int next;
    bool keep, report;
};

Out rules(int s, uint32_t k, uint32_t sync, uint32_t rel)
{
    using namespace hirace;
    const Desc d = kStates[s];
    const int ck = cls_low(k), gk = cls_grid(k);
    const int RW = ST_RACE_W, RB = ST_RACE_B, RG = ST_RACE_G;
    /* rule 0 */
    if (d.grp == G_RACE) {
        if (sync == SYNC_GS)
            return {s, true, false};
        if (s == RW && rel == REL_B && sync == SYNC_US)
            return {RB, true, true};
        if ((s == RW || s == RB) && rel == REL_G)
            return {RG, true, true};
        return {s, true, false};
    }
    /* rule 1 */
    if (d.grp == G_INIT || sync == SYNC_GS)
        return {find(G_T, ck, ck, gk), false, false};
    /* rule 2 */
    if (d.grp == G_G)
        return compatG(d.a, k) ? Out{s, true, false} : Out{RG, false, true};
    int KT = 0, KB = 0, KG = 0;
    if (d.grp == G_T) {
        KT = d.a;
        KB = d.b;
        KG = d.c;
    } else if (d.grp == G_W) {
        KT = d.a;
        KB = d.b;
        KG = d.c;
    } else { /* G_B */
        KB = d.a;
        KG = d.b;
    }
    const int KBp = join(KB, ck), KGp = join(KG, gk);
    /* rule 3 */
    if (rel == REL_G)
        return compatG(KG, k) ? Out{find(G_G, KG, 0, 0), false, false} : Out{RG, false, true};
    /* rule 4 */
    if (sync == SYNC_BS)
        return {find(G_T, ck, ck, KGp), false, false};
    /* rule 5 */
    if (d.grp == G_B)
        return compat(d.a, k) ? Out{find(G_B, d.a, KGp, 0), true, false} : Out{RB, false, true};
    /* rule 6 */
    if (rel == REL_B)
        return compat(KB, k) ? Out{find(G_B, KB, KGp, 0), false, false} : Out{RB, false, true};
    /* rule 7 */
    if (sync == SYNC_WS)
        return {find(G_T, ck, KBp, KGp), false, false};
    /* rule 8 */
    if (d.grp == G_W)
        return compat(d.a, k) ? Out{find(G_W, d.a, KBp, KGp), true, false} : Out{RW, false, true};
    /* rule 9 */
    if (rel == REL_W)
        return compat(KT, k) ? Out{find(G_W, KT, KBp, KGp), false, false} : Out{RW, false, true};
    /* rule 10 */
    return {find(G_T, join(KT, ck), KBp, KGp), true, false};
}

/* ---- relaxed read-vs-atomic policy (reading R2 alternative) ----
 * Conflicts: W with anything; across blocks AB-AB and AB-AG.  A plain read never conflicts with
 * an atomic, and atomics of one block never conflict.  Inside a block only W matters (classes
 * N = non-write, X = write).  Across blocks a block's kinds summarise into the chain
 * R < RAG (some AG) < RAB (some AB) < X (some W): a new R is compatible unless X, an AG only
 * with R/RAG, an AB only with R.  With >= 2 blocks and no race the configurations are:
 *   G_R   only reads;                       G_AG1 AG in exactly one block (the record's), R elsewhere;
 *   G_AGn AG in >= 2 blocks, R elsewhere;   G_AB1 AB (+ maybe AG) in exactly one block (the record's).
 * State codes keep INIT = 0 and RACE_W/B/G = 20/21/22. */
namespace relaxed {

enum { N = 0, X = 1 };
enum { GR = 0, GRAG = 1, GRAB = 2, GX = 3 };
enum { S_INIT = 0, T0 = 1, W0 = 7, B0 = 12, G_R = 16, G_AG1 = 17, G_AGn = 18, G_AB1 = 19 };

struct RDesc {
    Group grp;
    int a, b, c; /* T: KT, KB, KG   W: KB, KG   B: KG */
};

const RDesc kR[hirace::ST_COUNT] = {
    {G_INIT, 0, 0, 0},
    {G_T, N, N, GR},  {G_T, N, N, GRAG}, {G_T, N, N, GRAB}, {G_T, N, N, GX}, {G_T, N, X, GX}, {G_T, X, X, GX},
    {G_W, N, GR, 0},  {G_W, N, GRAG, 0}, {G_W, N, GRAB, 0}, {G_W, N, GX, 0}, {G_W, X, GX, 0},
    {G_B, GR, 0, 0},  {G_B, GRAG, 0, 0}, {G_B, GRAB, 0, 0}, {G_B, GX, 0, 0},
    {G_G, 0, 0, 0},   {G_G, 1, 0, 0},    {G_G, 2, 0, 0},    {G_G, 3, 0, 0},
    {G_RACE, 1, 0, 0}, {G_RACE, 2, 0, 0}, {G_RACE, 3, 0, 0},
};

int clsL(uint32_t k) { return k == HIRACE_WRITE ? X : N; }
int clsG(uint32_t k)
{
    return k == HIRACE_READ ? GR : (k == HIRACE_ATOMIC_GRID ? GRAG : (k == HIRACE_ATOMIC_BLOCK ? GRAB : GX));
}
int jmax(int x, int y) { return x > y ? x : y; }

int findT(int kt, int kb, int kg)
{
    for (int s = T0; s < W0; s++)
        if (kR[s].a == kt && kR[s].b == kb && kR[s].c == kg)
            return s;
    return -1;
}
int findW(int kb, int kg)
{
    for (int s = W0; s < B0; s++)
        if (kR[s].a == kb && kR[s].b == kg)
            return s;
    return -1;
}
int findB(int kg) { return B0 + kg; }

Out rules(int s, uint32_t k, uint32_t sync, uint32_t rel)
{
    using namespace hirace;
    const RDesc d = kR[s];
    const int RW = ST_RACE_W, RB = ST_RACE_B, RG = ST_RACE_G;
    /* rule 0: RACE records are frozen; class upgrades inside the first racing epoch */
    if (d.grp == G_RACE) {
        if (sync == SYNC_GS)
            return {s, true, false};
        if (s == RW && rel == REL_B && sync == SYNC_US)
            return {RB, true, true};
        if ((s == RW || s == RB) && rel == REL_G)
            return {RG, true, true};
        return {s, true, false};
    }
    /* rule 1 */
    if (d.grp == G_INIT || sync == SYNC_GS)
        return {findT(clsL(k), clsL(k), clsG(k)), false, false};
    const bool same = rel != REL_G;
    /* rule 2: >= 2 blocks in the grid epoch */
    if (d.grp == G_G) {
        if (k == HIRACE_WRITE)
            return {RG, false, true};
        switch (s) {
        case G_R:
            if (k == HIRACE_READ)
                return {G_R, true, false};
            return {k == HIRACE_ATOMIC_GRID ? G_AG1 : G_AB1, false, false}; /* record := the atomic's block */
        case G_AG1:
            if (k == HIRACE_READ)
                return {G_AG1, true, false};
            if (k == HIRACE_ATOMIC_GRID)
                return {same ? G_AG1 : G_AGn, true, false};
            return same ? Out{G_AB1, true, false} : Out{RG, false, true}; /* AB */
        case G_AGn:
            if (k == HIRACE_ATOMIC_BLOCK)
                return {RG, false, true};
            return {G_AGn, true, false};
        default: /* G_AB1 */
            if (k == HIRACE_READ || same)
                return {G_AB1, true, false};
            return {RG, false, true};
        }
    }
    int KT = N, KB, KG;
    if (d.grp == G_T) {
        KT = d.a;
        KB = d.b;
        KG = d.c;
    } else if (d.grp == G_W) {
        KB = d.a;
        KG = d.b;
    } else { /* B */
        KB = N;
        KG = d.a;
    }
    const int cl = clsL(k), cg = clsG(k);
    const int KBp = jmax(KB, cl), KGp = jmax(KG, cg);
    /* rule 3: first access of another block in this grid epoch */
    if (rel == REL_G) {
        if (k == HIRACE_WRITE || KG == GX)
            return {RG, false, true};
        if (k == HIRACE_READ)
            return KG == GR ? Out{G_R, false, false} : Out{KG == GRAG ? G_AG1 : G_AB1, true, false};
        if (k == HIRACE_ATOMIC_GRID)
            return KG == GR ? Out{G_AG1, false, false} : (KG == GRAG ? Out{G_AGn, true, false} : Out{RG, false, true});
        return KG == GR ? Out{G_AB1, false, false} : Out{RG, false, true}; /* AB */
    }
    /* rule 4 */
    if (sync == SYNC_BS)
        return {findT(cl, cl, KGp), false, false};
    /* rule 5 */
    if (d.grp == G_B)
        return k != HIRACE_WRITE ? Out{findB(KGp), true, false} : Out{RB, false, true};
    /* rule 6 */
    if (rel == REL_B)
        return (KB == N && k != HIRACE_WRITE) ? Out{findB(KGp), false, false} : Out{RB, false, true};
    /* rule 7 */
    if (sync == SYNC_WS)
        return {findT(cl, KBp, KGp), false, false};
    /* rule 8 */
    if (d.grp == G_W)
        return k != HIRACE_WRITE ? Out{findW(KBp, KGp), true, false} : Out{RW, false, true};
    /* rule 9 */
    if (rel == REL_W)
        return (KT == N && k != HIRACE_WRITE) ? Out{findW(KBp, KGp), false, false} : Out{RW, false, true};
    /* rule 10 */
    return {findT(jmax(KT, cl), KBp, KGp), true, false};
}

} // namespace relaxed

/* ---- cluster level (reading R16) ---------------------------------
 * thread < warp < block < cluster < grid.  Across blocks (of one cluster or of two clusters)
 * the grid classes apply (clsG); inside a block the low classes (cls).  States:
 *   T(KT,KB,KC,KG)  one thread in the current warp epoch; KC = its block's kinds in the cluster
 *                   epoch, KG = its cluster's kinds in the grid epoch (grid classes)
 *   W(c,KB,KC,KG)   >= 2 threads of one warp;   B(c,KC,KG) >= 2 warps of one block
 *   C(c,KG)         >= 2 blocks of one cluster in the cluster epoch, all of grid class c
 *   G(c)            >= 2 clusters in the grid epoch
 *   RACE_W/B/G/C    class codes 1/2/3/4 (the oracle's), sticky, frozen record
 * Rules, first match wins (record := the accessor unless "keep"); KB' = join(KB, cls k),
 * KC' = join(KC, clsG k), KG' = join(KG, clsG k):
 *   0 RACE: Gs keep; RACE_W & rel B & Us -> RACE_B; RACE_W/B & rel C & Us -> RACE_C;
 *     RACE_W/B/C & rel G & !Gs -> RACE_G (upgrades report, keep); otherwise keep
 *   1 INIT or Gs -> T(cls k, cls k, clsG k, clsG k)
 *   2 G(c): compatG(c,k) -> keep, else RACE_G          3 rel G: compatG(KG,k) -> G(KG), else RACE_G
 *   4 Cs -> T(cls k, cls k, clsG k, KG')
 *   5 C(c,KG): compatG(c,k) -> C(c,KG') keep, else RACE_C
 *   6 rel C: compatG(KC,k) -> C(KC,KG'), else RACE_C
 *   7 Bs -> T(cls k, cls k, KC', KG')
 *   8 B(c,KC,KG): compat(c,k) -> B(c,KC',KG') keep, else RACE_B
 *   9 rel B: compat(KB,k) -> B(KB,KC',KG'), else RACE_B
 *  10 Ws -> T(cls k, KB', KC', KG')
 *  11 W(c,..): compat(c,k) -> W(c,KB',KC',KG') keep, else RACE_W
 *  12 rel W: compat(KT,k) -> W(KT,KB',KC',KG'), else RACE_W
 *  13 rel S: T(join(KT, cls k), KB', KC', KG') keep
 * The state list is the set reachable from INIT, sorted by (group, fields), RACE states last. */
namespace clus {

using namespace hirace::cluster;
enum CGroup { Q_INIT = 0, Q_T, Q_W, Q_B, Q_C, Q_G, Q_RACE };
struct CD {
    int grp, a, b, c, d; /* T: KT,KB,KC,KG  W: c,KB,KC,KG  B: c,-,KC,KG  C: c,-,-,KG  G: c  RACE: class */
    bool operator==(const CD &o) const { return grp == o.grp && a == o.a && b == o.b && c == o.c && d == o.d; }
    bool operator<(const CD &o) const
    {
        if (grp != o.grp) return grp < o.grp;
        if (a != o.a) return a < o.a;
        if (b != o.b) return b < o.b;
        if (c != o.c) return c < o.c;
        return d < o.d;
    }
};
struct COut {
    CD next;
    bool keep, report;
};
const CD INIT{Q_INIT, 0, 0, 0, 0};
CD T(int kt, int kb, int kc, int kg) { return {Q_T, kt, kb, kc, kg}; }
CD Wq(int c, int kb, int kc, int kg) { return {Q_W, c, kb, kc, kg}; }
CD Bq(int c, int kc, int kg) { return {Q_B, c, 0, kc, kg}; }
CD Cq(int c, int kg) { return {Q_C, c, 0, 0, kg}; }
CD Gq(int c) { return {Q_G, c, 0, 0, 0}; }
CD RACE(int cls) { return {Q_RACE, cls, 0, 0, 0}; }
enum { RW = 1, RB = 2, RG = 3, RC = 4 };

COut rules(const CD &d, uint32_t k, uint32_t sync, uint32_t rel)
{
    const int ck = cls_low(k), gk = cls_grid(k);
    if (d.grp == Q_RACE) { /* rule 0 */
        if (sync == SYNC_GS)
            return {d, true, false};
        if (d.a == RW && rel == REL_B && sync == SYNC_US)
            return {RACE(RB), true, true};
        if ((d.a == RW || d.a == RB) && rel == REL_C && sync == SYNC_US)
            return {RACE(RC), true, true};
        if (d.a != RG && rel == REL_G)
            return {RACE(RG), true, true};
        return {d, true, false};
    }
    if (d.grp == Q_INIT || sync == SYNC_GS) /* rule 1 */
        return {T(ck, ck, gk, gk), false, false};
    if (d.grp == Q_G) /* rule 2 */
        return compatG(d.a, k) ? COut{d, true, false} : COut{RACE(RG), false, true};
    const int KT = d.a, KB = d.grp == Q_B ? d.a : d.b, KC = d.grp == Q_C ? d.a : d.c, KG = d.d;
    const int KBp = join(KB, ck), KCp = join(KC, gk), KGp = join(KG, gk);
    if (rel == REL_G) /* rule 3 */
        return compatG(KG, k) ? COut{Gq(KG), false, false} : COut{RACE(RG), false, true};
    if (sync == SYNC_CS) /* rule 4 */
        return {T(ck, ck, gk, KGp), false, false};
    if (d.grp == Q_C) /* rule 5 */
        return compatG(d.a, k) ? COut{Cq(d.a, KGp), true, false} : COut{RACE(RC), false, true};
    if (rel == REL_C) /* rule 6 */
        return compatG(KC, k) ? COut{Cq(KC, KGp), false, false} : COut{RACE(RC), false, true};
    if (sync == SYNC_BS) /* rule 7 */
        return {T(ck, ck, KCp, KGp), false, false};
    if (d.grp == Q_B) /* rule 8 */
        return compat(d.a, k) ? COut{Bq(d.a, KCp, KGp), true, false} : COut{RACE(RB), false, true};
    if (rel == REL_B) /* rule 9 */
        return compat(KB, k) ? COut{Bq(KB, KCp, KGp), false, false} : COut{RACE(RB), false, true};
    if (sync == SYNC_WS) /* rule 10 */
        return {T(ck, KBp, KCp, KGp), false, false};
    if (d.grp == Q_W) /* rule 11 */
        return compat(d.a, k) ? COut{Wq(d.a, KBp, KCp, KGp), true, false} : COut{RACE(RW), false, true};
    if (rel == REL_W) /* rule 12 */
        return compat(KT, k) ? COut{Wq(KT, KBp, KCp, KGp), false, false} : COut{RACE(RW), false, true};
    return {T(join(KT, ck), KBp, KCp, KGp), true, false}; /* rule 13 */
}

/* reachable states from INIT under every label, sorted; RACE states sort last by group */
int states(CD *out, int cap)
{
    int n = 0;
    out[n++] = INIT;
    for (int i = 0; i < n; i++)
        for (uint32_t k = 0; k < 4; k++)
            for (uint32_t y = 0; y < 5; y++)
                for (uint32_t r = 0; r < 5; r++) {
                    const CD nx = rules(out[i], k, y, r).next;
                    bool seen = false;
                    for (int j = 0; j < n && !seen; j++)
                        seen = out[j] == nx;
                    if (!seen) {
                        if (n == cap)
                            return -1;
                        out[n++] = nx;
                    }
                }
    for (int i = 1; i < n; i++) /* insertion sort (INIT stays first: group 0) */
        for (int j = i; j > 0 && out[j] < out[j - 1]; j--) {
            CD t = out[j];
            out[j] = out[j - 1];
            out[j - 1] = t;
        }
    return n;
}

} // namespace clus

} // namespace

namespace hirace_impl {
/* masked replay (subwarp.cu): a race the sub-warp history finds has the level of the state the
 * FSM reached -- one warp (T, W) -> RACE_W, >= 2 warps (B) -> RACE_B, >= 2 blocks (G) -> RACE_G */
void fsm_race_of(int policy, unsigned char out[32])
{
    for (int s = 0; s < 32; s++) {
        Group g = G_NONE;
        if (s < (int)hirace::ST_COUNT)
            g = policy == 1 ? relaxed::kR[s].grp : kStates[s].grp;
        out[s] = (unsigned char)(g == G_T || g == G_W ? hirace::ST_RACE_W
                                                       : g == G_B ? hirace::ST_RACE_B
                                                                  : g == G_G ? hirace::ST_RACE_G : s);
    }
}
} // namespace hirace_impl

extern "C" hirace_status hirace_fsm_table_policy(int policy, unsigned char out[2048])
{
    if (!out || policy < 0 || policy > 1)
        return HIRACE_E_INVAL;
    for (int s = 0; s < 32; s++) {
        for (uint32_t k = 0; k < 4; k++)
            for (uint32_t y = 0; y < 4; y++)
                for (uint32_t r = 0; r < 4; r++) {
                    uint32_t idx = ((uint32_t)s << 6) | (k << 4) | (y << 2) | r;
                    if (s >= (int)hirace::ST_COUNT) {
                        out[idx] = (unsigned char)(s | hirace::E_KEEP); /* unused codes */
                        continue;
                    }
                    Out o = policy == 0 ? rules(s, k, y, r) : relaxed::rules(s, k, y, r);
                    if (o.next < 0)
                        return HIRACE_E_INVAL; /* inconsistent tuple: a rule-table bug */
                    out[idx] = (unsigned char)(o.next | (o.keep ? hirace::E_KEEP : 0) |
                                               (o.report ? hirace::E_REPORT : 0));
                }
    }
    return HIRACE_OK;
}

extern "C" hirace_status hirace_fsm_table(unsigned char out[2048]) { return hirace_fsm_table_policy(0, out); }

extern "C" uint64_t hirace_fsm_step_policy(int policy, uint64_t old_shadow, uint32_t tid, uint32_t kind, uint32_t g,
                                           uint32_t b, uint32_t w, uint32_t block_threads, uint32_t warp_size,
                                           int *report)
{
    static unsigned char tables[2][2048];
    static bool built[2] = {false, false};
    policy = policy == 1 ? 1 : 0;
    if (!built[policy]) {
        hirace_fsm_table_policy(policy, tables[policy]);
        built[policy] = true;
    }
    const unsigned char *table = tables[policy];
    hirace_dev_ctx c{};
    c.block_threads = block_threads ? block_threads : 1;
    c.warp_size = warp_size ? warp_size : 1;
    hirace::fastdiv_init(c.block_threads, &c.bt_magic, &c.bt_s1, &c.bt_s2);
    hirace::fastdiv_init(c.warp_size, &c.ws_magic, &c.ws_s1, &c.ws_s2);
    const hirace::geom G = hirace::make_geom(c);
    hirace::access a;
    a.tid = tid;
    a.kind = kind & 3;
    a.g = g;
    a.b = b;
    a.w = w;
    uint32_t rep = 0;
    uint64_t n = hirace::step(old_shadow, a, table, G, &rep);
    if (report)
        *report = (int)rep;
    return n;
}

extern "C" uint64_t hirace_fsm_step(uint64_t old_shadow, uint32_t tid, uint32_t kind, uint32_t g, uint32_t b,
                                    uint32_t w, uint32_t block_threads, uint32_t warp_size, int *report)
{
    return hirace_fsm_step_policy(0, old_shadow, tid, kind, g, b, w, block_threads, warp_size, report);
}

/* compact 4-byte record (hirace_shadow_alloc_compact): the kernels' raw-flag table and
 * label_raw_c / next_c, on the host */
extern "C" uint32_t hirace_fsm_step_compact(int policy, uint32_t old_shadow, uint32_t tid, uint32_t kind, uint32_t g,
                                            uint32_t b, uint32_t w, uint32_t block_threads, uint32_t warp_size,
                                            uint32_t grid_threads, const hirace_epoch_limits *lim, int *report)
{
    static unsigned char raw[2][2048 + hirace::RAW_TABLE_BYTES];
    static bool built[2] = {false, false};
    policy = policy == 1 ? 1 : 0;
    if (!built[policy]) {
        hirace_fsm_table_policy(policy, raw[policy]);
        hirace::expand_raw_table(raw[policy], raw[policy] + 2048);
        built[policy] = true;
    }
    hirace::clay L;
    if (!lim || !hirace::make_clay(lim->max_g, lim->max_b, lim->max_w, grid_threads, &L))
        return 0xffffffffu;
    hirace_dev_ctx c{};
    c.block_threads = block_threads ? block_threads : 1;
    c.warp_size = warp_size ? warp_size : 1;
    hirace::fastdiv_init(c.block_threads, &c.bt_magic, &c.bt_s1, &c.bt_s2);
    hirace::fastdiv_init(c.warp_size, &c.ws_magic, &c.ws_s1, &c.ws_s2);
    const hirace::geom G = hirace::make_geom(c);
    uint32_t rep = 0;
    const uint32_t n = hirace::step_c(old_shadow, tid, kind & 3u, hirace::c_epochs(L, g, b, w), raw[policy] + 2048, L,
                                      G, &rep);
    if (report)
        *report = (int)rep;
    return n;
}

/* Cluster-level table (hirace::cluster layout): 64 states x 256 labels. */
extern "C" hirace_status hirace_fsm_table_cluster(unsigned char out[16384], uint32_t *n_states)
{
    using namespace clus;
    if (!out)
        return HIRACE_E_INVAL;
    CD st[64];
    const int n = states(st, 64);
    if (n < 0)
        return HIRACE_E_INVAL; /* more than 64 states: a rule bug */
    memset(out, 0, 16384);
    for (int s = 0; s < 64; s++)
        for (uint32_t lab = 0; lab < 256; lab++) {
            const uint32_t k = lab >> 6, y = (lab >> 3) & 7u, r = lab & 7u;
            const uint32_t idx = ((uint32_t)s << 8) | lab;
            if (s >= n || y > 4 || r > 4) {
                out[idx] = (unsigned char)(s | E_KEEP); /* unused codes */
                continue;
            }
            const COut o = rules(st[s], k, y, r);
            int nx = -1;
            for (int j = 0; j < n; j++)
                if (st[j] == o.next)
                    nx = j;
            if (nx < 0)
                return HIRACE_E_INVAL;
            out[idx] = (unsigned char)(nx | (o.keep ? E_KEEP : 0) | (o.report ? E_REPORT : 0));
        }
    if (n_states)
        *n_states = (uint32_t)n;
    return HIRACE_OK;
}

/* Race class of a cluster-table state code (0 if not RACE): WARP 1, BLOCK 2, GRID 3, CLUSTER 4. */
extern "C" uint32_t hirace_fsm_cluster_class(uint32_t state)
{
    using namespace clus;
    CD st[64];
    const int n = states(st, 64);
    if (n < 0 || state >= (uint32_t)n || st[state].grp != Q_RACE)
        return 0;
    return (uint32_t)st[state].a;
}

extern "C" uint64_t hirace_fsm_step_cluster(uint64_t old_shadow, uint32_t tid, uint32_t kind, uint32_t g, uint32_t c,
                                            uint32_t b, uint32_t w, uint32_t block_threads, uint32_t warp_size,
                                            uint32_t cluster_blocks, int *report)
{
    static unsigned char table[16384];
    static bool built = false;
    if (!built) {
        hirace_fsm_table_cluster(table, nullptr);
        built = true;
    }
    if (!block_threads || !warp_size || !cluster_blocks || g > hirace::cluster::MAX_G ||
        c > hirace::cluster::MAX_C || b > hirace::cluster::MAX_B || w > hirace::cluster::MAX_W ||
        tid > hirace::cluster::MAX_TID)
        return ~0ull;
    uint32_t rep = 0;
    const uint64_t n = hirace::cluster::step(old_shadow, tid, kind & 3u, g, c, b, w, table, block_threads, warp_size,
                                             cluster_blocks, &rep);
    if (report)
        *report = (int)rep;
    return n;
}
