/*
 * include/prng_device.cuh — header-only device side of the expander-walk PRNG.
 *
 *   prng_next(&state)  = Alg.2 GetNextRand (§III-B) called by any
 *   GPU thread "at any point of time" (§III): l = 64 steps of the walk on
 *   the 7-regular Gabber–Galil expander (§III-A), 3 bits per step, and
 *   the walker's vertex label returned as a 64-bit number (§III-B).
 *
 * Usage inside a user kernel (after prng_epoch_begin + prng_device_view;
 * pass the view as a __grid_constant__ kernel parameter):
 *     prng_state st = prng_state_load(&view, slot);   // slot = walker by default
 *     uint64_t r = prng_next(&st);             // as often as the epoch allows
 *     prng_state_store(&view, &st);
 * prng_next(&st, &view) is the same call with the view named explicitly, and
 * prng_next<PRNG_WALK_L64>(...) compiles in only the paper's l = 64, m = 2^k
 * walk (the host picks the mode with prng_walk_mode(&view); see below).
 * A walker must be used by one thread at a time (that is what makes the
 * generator thread-safe, §I-B).  A draw outside the epoch window sets a
 * sticky flag (read by prng_check) and returns 0 — never different bits.
 *
 * This header is part of the GPU path.  It shares nothing with oracle/.
 */
#ifndef GGPRNG_PRNG_DEVICE_CUH
#define GGPRNG_PRNG_DEVICE_CUH

#include <stdint.h>

#define PRNG_FLAG_OVERRUN 1u

/* Everything a device thread needs; filled by prng_device_view(). */
struct prng_view {
    const uint32_t *bits;  /* epoch window, SoA: word (d*R + r) of window slot k at bits[(d*R+r)*pitch + k] */
    const uint32_t *wmap;  /* slot -> walker (prng_epoch_begin_list), or NULL: slot k = walker k */
    uint32_t *x;           /* walker vertex, x coordinate (wrapped mod 2^32 when m is a power of two) */
    uint32_t *y;           /* walker vertex, y coordinate */
    uint32_t *j;           /* next absolute draw index of each walker */
    uint32_t *flags;       /* sticky error flags (PRNG_FLAG_*) */
    uint64_t pitch;        /* words between rows of the window */
    uint64_t m;            /* modulus */
    uint32_t J0;           /* first draw of the window */
    uint32_t D;            /* draws per walker in the window */
    uint32_t Wv;           /* slots covered by the window: [0, Wv) */
    uint32_t R;            /* words per draw record = ceil(3l/32) */
    uint32_t l;            /* steps per number */
    uint32_t log2m;        /* log2(m) if m is a power of two, else 0 */
    uint32_t pow2;         /* 1 if m is a power of two */
    uint32_t variant;      /* 0 = forward maps; 1 = bipartite (sigma / sigma^-1 alternating) */
    uint32_t l0;           /* burn-in steps (global step parity for variant 1) */
    uint32_t _pad;
    const uint32_t *tab;   /* composed-step table in global memory (PRNG_TABLE_WORDS words) */
};

struct prng_state {
    uint32_t x, y;     /* current vertex */
    uint32_t walker;   /* walker id (handle-local): index of the state arrays */
    uint32_t slot;     /* column of the epoch window holding this walker's bits */
    uint32_t used;     /* draws consumed in this epoch */
    const struct prng_view *view;  /* the view it was loaded from (one-argument prng_next) */
};

/* ------------------------------------------------------------------------
 * The Gabber–Galil step (§III-A), 3-bit choice b, k = b mod 7 (R4):
 *   b in {1,2,3}: y <- y + 2x + (b-1)        (sigma_1..3)
 *   b in {4,5,6}: x <- x + 2y + (b-4)        (sigma_4..6)
 *   b in {0,7}  : stay                        (sigma_0)
 * For m = 2^k all arithmetic is done in Z/2^32 and reduced at emission
 * (Z/2^32 -> Z/2^k is a ring homomorphism).
 *
 * Fast form (l = 64).  The 192-bit record is repacked into 7 words of 10
 * whole 3-bit fields (no field straddles a word).  Per word, SWAR gives
 *   MY = fields in {1,2,3}, MX = fields in {4,5,6} (bit at the field's LSB),
 *   C  = field - [y-move], whose low two bits are the step's constant c.
 * With u = x + y + c both moves are one add:  y-move y' = u + x,
 * x-move x' = u + y.  Per step 7 SASS, which ptxas splits evenly between
 * the ALU pipe and the FMA-heavy pipe (IMAD.*); on sm_100a each accepts a
 * warp instruction every other cycle per SMSP, so a 50/50 split is what lets
 * the scheduler issue every cycle:
 *   LOP3.P py, LOP3.P px        predicates from MY / MX              (ALU)
 *   IMAD.SHL ct = C << (30-3k)  c to the top two bits                (FMA)
 *   s = x + y ; LEA.HI u = s + (ct >> 30)                            (FMA, ALU)
 *   @py y = u + x ; @px x = u + y                                    (ALU / FMA)
 * ------------------------------------------------------------------------ */
template <int K>
__device__ __forceinline__ void gg_step_swar(uint32_t MY, uint32_t MX, uint32_t C,
                                             uint32_t &x, uint32_t &y)
{
    asm volatile(
        "{\n\t"
        ".reg .pred py, px;\n\t"
        ".reg .b32 ty, tx, ct, c, s, u;\n\t"
        "and.b32 ty, %2, %5;\n\t"
        "setp.ne.b32 py, ty, 0;\n\t"
        "and.b32 tx, %3, %5;\n\t"
        "setp.ne.b32 px, tx, 0;\n\t"
        "shl.b32 ct, %4, %6;\n\t"
        "shr.b32 c, ct, 30;\n\t"
        "add.u32 s, %0, %1;\n\t"
        "add.u32 u, s, c;\n\t"
        "@py add.u32 %1, u, %0;\n\t"
        "@px add.u32 %0, u, %1;\n\t"
        "}"
        : "+r"(x), "+r"(y)
        : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3 * K)), "n"(30 - 3 * K));
}

template <int NK>
__device__ __forceinline__ void gg_word10(uint32_t Q, uint32_t &x, uint32_t &y)
{
    const uint32_t f1 = Q >> 1, f2 = Q >> 2;
    /* MY: b2=0 and b != 0, kept only at the fields' LSBs (it is subtracted
     * below); MX: b2=1 and b != 7 (only its LSB bits are ever tested) */
    const uint32_t MY = ((f1 | Q) & 0x09249249u) & ~f2;
    const uint32_t MX = f2 & ~(f1 & Q);
    /* y-move fields hold b-1 (no borrow: b>=1) */
    const uint32_t C = Q - MY;
    if (NK > 0) gg_step_swar<0>(MY, MX, C, x, y);
    if (NK > 1) gg_step_swar<1>(MY, MX, C, x, y);
    if (NK > 2) gg_step_swar<2>(MY, MX, C, x, y);
    if (NK > 3) gg_step_swar<3>(MY, MX, C, x, y);
    if (NK > 4) gg_step_swar<4>(MY, MX, C, x, y);
    if (NK > 5) gg_step_swar<5>(MY, MX, C, x, y);
    if (NK > 6) gg_step_swar<6>(MY, MX, C, x, y);
    if (NK > 7) gg_step_swar<7>(MY, MX, C, x, y);
    if (NK > 8) gg_step_swar<8>(MY, MX, C, x, y);
    if (NK > 9) gg_step_swar<9>(MY, MX, C, x, y);
}

/* 64 steps from a 6-word record, m = 2^k (wrapped arithmetic). */
__device__ __forceinline__ void gg_walk64(const uint32_t w[6], uint32_t &x, uint32_t &y)
{
    gg_word10<10>(w[0], x, y);
    gg_word10<10>(__funnelshift_r(w[0], w[1], 30), x, y);
    gg_word10<10>(__funnelshift_r(w[1], w[2], 28), x, y);
    gg_word10<10>(__funnelshift_r(w[2], w[3], 26), x, y);
    gg_word10<10>(__funnelshift_r(w[3], w[4], 24), x, y);
    gg_word10<10>(__funnelshift_r(w[4], w[5], 22), x, y);
    gg_word10<4>(w[5] >> 20, x, y);
}

/* Read-only 32-bit load that the compiler may not sink below later volatile
 * asm (the walk): used to prefetch the next draw's record a full walk ahead. */
__device__ __forceinline__ uint32_t gg_ldg_early(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

/* Two independent walkers interleaved step by step (more ILP per warp:
 * the scheduler always has an instruction of the other walker ready). */
template <int NK>
__device__ __forceinline__ void gg_word10x2(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                            uint32_t &xb, uint32_t &yb)
{
    const uint32_t f1a = Qa >> 1, f2a = Qa >> 2, f1b = Qb >> 1, f2b = Qb >> 2;
    const uint32_t MYa = ((f1a | Qa) & 0x09249249u) & ~f2a, MXa = f2a & ~(f1a & Qa);
    const uint32_t MYb = ((f1b | Qb) & 0x09249249u) & ~f2b, MXb = f2b & ~(f1b & Qb);
    const uint32_t Ca = Qa - MYa, Cb = Qb - MYb;
#define GG_S2(k)                                               \
    if (NK > k) {                                              \
        gg_step_swar<k>(MYa, MXa, Ca, xa, ya);                 \
        gg_step_swar<k>(MYb, MXb, Cb, xb, yb);                 \
    }
    GG_S2(0) GG_S2(1) GG_S2(2) GG_S2(3) GG_S2(4) GG_S2(5) GG_S2(6) GG_S2(7) GG_S2(8) GG_S2(9)
#undef GG_S2
}

__device__ __forceinline__ void gg_walk64x2(const uint32_t a[6], const uint32_t b[6], uint32_t &xa,
                                            uint32_t &ya, uint32_t &xb, uint32_t &yb)
{
    gg_word10x2<10>(a[0], b[0], xa, ya, xb, yb);
    gg_word10x2<10>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb);
    gg_word10x2<10>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb);
    gg_word10x2<10>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb);
    gg_word10x2<10>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb);
    gg_word10x2<10>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb);
    gg_word10x2<4>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb);
}

/* ------------------------------------------------------------------------
 * R2P form of the same step (default for l = 64, m = 2^k).  The per-step
 * predicate tests (two LOP3.P per step above) are replaced by loading the
 * predicate register file from one byte of a flag word: ptxas turns four
 * single-bit tests of the same register that fall inside one byte into one
 * R2P PR, F.Bn (measured, tools/step_bench2.cu).  Per 10-field word:
 *   F = MY at field bit 0 (y-move) | MX at field bit 1 (x-move),  G = F >> 4
 * and the 10 steps are grouped in pairs so that each pair's four flags sit in
 * bits 0..6 of one byte of F or G (step k's flags: F bits 3k, 3k+1):
 *   F.B0 steps 0,1 | G.B0 steps 2,3 | G.B1 steps 4,5 | F.B2 steps 6,7 |
 *   F.B3 steps 8,9                          (4-field tail word: F.B0 | G.B0)
 * i.e. 5 R2P + 1 shift per 10 steps instead of 20 LOP3.P (with G = F >> 6 no
 * pairing covers all ten steps: 6 R2P).  The arithmetic is
 * unchanged (u = x + y + c; y' = u + x | x' = u + y), so both forms are the
 * same evaluation of the paper's step.
 * ------------------------------------------------------------------------ */
#define GG_R2P_U(S)                                                                   \
    "shl.b32 ct, %3, " S ";\n\tshr.b32 c, ct, 30;\n\tadd.u32 s, %0, %1;\n\tadd.u32 u, s, c;\n\t"

/* Two steps: py/px of the first at bits B0/B0+1 of S, of the second at B1/B1+1;
 * SH0/SH1 = 30 - 3k bring field k's constant to the top of C. */
template <int B0, int B1, int SH0, int SH1>
__device__ __forceinline__ void gg_r2p_two(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y)
{
    asm volatile(
        "{\n\t.reg .pred py0, px0, py1, px1;\n\t.reg .b32 t, ct, c, u, s;\n\t"
        "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
        "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
        "and.b32 t, %2, %6;\n\tsetp.ne.b32 py1, t, 0;\n\t"
        "and.b32 t, %2, %7;\n\tsetp.ne.b32 px1, t, 0;\n\t"
        GG_R2P_U("%8") "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t"
        GG_R2P_U("%9") "@py1 add.u32 %1, u, %0;\n\t@px1 add.u32 %0, u, %1;\n\t}"
        : "+r"(x), "+r"(y)
        : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(1u << B1), "n"(2u << B1), "n"(SH0),
          "n"(SH1));
}

/* Bipartite walk (variant 1): a pair of steps whose first
 * (even global step) applies sigma_k and whose second (odd) applies
 * sigma_k^{-1}: y' = y - 2x - c | x' = x - 2y - c, as r = 2x + c, v = 2y + c
 * (IMAD), @py y -= r, @px x -= v: 6 SASS instead of 5, kept on the FMA-heavy
 * pipe where it can be (the plain-add form put 2/3 of the kernel on the ALU). */
#define GG_R2P_INV(S)                                                                      \
    "shl.b32 ct, %3, " S ";\n\tshr.b32 c, ct, 30;\n\t"                                      \
    "mad.lo.u32 r, %0, 2, c;\n\tmad.lo.u32 v, %1, 2, c;\n\t"

template <int B0, int B1, int SH0, int SH1>
__device__ __forceinline__ void gg_r2p_two_bip(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y)
{
    asm volatile(
        "{\n\t.reg .pred py0, px0, py1, px1;\n\t.reg .b32 t, ct, c, u, s, r, v;\n\t"
        "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
        "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
        "and.b32 t, %2, %6;\n\tsetp.ne.b32 py1, t, 0;\n\t"
        "and.b32 t, %2, %7;\n\tsetp.ne.b32 px1, t, 0;\n\t"
        GG_R2P_U("%8") "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t"
        GG_R2P_INV("%9") "@py1 sub.u32 %1, %1, r;\n\t@px1 sub.u32 %0, %0, v;\n\t}"
        : "+r"(x), "+r"(y)
        : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(1u << B1), "n"(2u << B1), "n"(SH0),
          "n"(SH1));
}

/* Flag word F and constant word C of a 10-field word Q (fields at 3i). */
__device__ __forceinline__ void gg_r2p_prep(uint32_t Q, uint32_t &C, uint32_t &F)
{
    const uint32_t f1 = Q >> 1, f2 = Q >> 2;
    const uint32_t MY = ((f1 | Q) & 0x09249249u) & ~f2; /* b in {1,2,3}, at 3i  */
    const uint32_t MX = f2 & ~(f1 & Q);                  /* b in {4,5,6}, at 3i (+garbage) */
    C = Q - MY;
    F = MY | ((MX << 1) & 0x12492492u);                  /* MX moved to 3i+1   */
}

#define GG_SH(k) (30 - 3 * (k))

/* A pair of steps (fields K, K+1 with flags at bits B0, B1 of S). */
template <bool BIP, int B0, int B1, int K>
__device__ __forceinline__ void gg_r2p_pair(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y)
{
    if (BIP)
        gg_r2p_two_bip<B0, B1, GG_SH(K), GG_SH(K + 1)>(S, C, x, y);
    else
        gg_r2p_two<B0, B1, GG_SH(K), GG_SH(K + 1)>(S, C, x, y);
}

template <int NK, bool BIP = false>
__device__ __forceinline__ void gg_word10_r2p(uint32_t Q, uint32_t &x, uint32_t &y)
{
    uint32_t C, F;
    gg_r2p_prep(Q, C, F);
    const uint32_t G = F >> 4;
    gg_r2p_pair<BIP, 0, 3, 0>(F, C, x, y);
    gg_r2p_pair<BIP, 2, 5, 2>(G, C, x, y);
    if (NK == 4) return;
    gg_r2p_pair<BIP, 8, 11, 4>(G, C, x, y);
    gg_r2p_pair<BIP, 18, 21, 6>(F, C, x, y);
    gg_r2p_pair<BIP, 24, 27, 8>(F, C, x, y);
}

/* Steps of one 10-field word (NK = 10) or of the 4-field tail word (NK = 4) for
 * two walkers, from prepared (C, F) of each. */
template <int NK, bool BIP = false>
__device__ __forceinline__ void gg_steps10x2_r2p(uint32_t Ca, uint32_t Fa, uint32_t Cb, uint32_t Fb,
                                                 uint32_t &xa, uint32_t &ya, uint32_t &xb, uint32_t &yb)
{
    const uint32_t Ga = Fa >> 4, Gb = Fb >> 4;
#define GG_R2P2(B0, B1, K0, K1, SA, SB)                                     \
    gg_r2p_pair<BIP, B0, B1, K0>(SA, Ca, xa, ya);                            \
    gg_r2p_pair<BIP, B0, B1, K0>(SB, Cb, xb, yb);
    GG_R2P2(0, 3, 0, 1, Fa, Fb)
    GG_R2P2(2, 5, 2, 3, Ga, Gb)
    if (NK == 4) return;
    GG_R2P2(8, 11, 4, 5, Ga, Gb)
    GG_R2P2(18, 21, 6, 7, Fa, Fb)
    GG_R2P2(24, 27, 8, 9, Fa, Fb)
#undef GG_R2P2
}

template <int NK, bool BIP = false>
__device__ __forceinline__ void gg_word10x2_r2p(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                                uint32_t &xb, uint32_t &yb)
{
    uint32_t Ca, Fa, Cb, Fb;
    gg_r2p_prep(Qa, Ca, Fa);
    gg_r2p_prep(Qb, Cb, Fb);
    gg_steps10x2_r2p<NK, BIP>(Ca, Fa, Cb, Fb, xa, ya, xb, yb);
}

/* R2P pair for m not a power of two, m <= 2^30 (x, y < m): u = x + y + c,
 * v = u + (py ? x : y) < 3m + 2 reduced by two conditional subtracts, then
 * stored into y or x by predicate (11 SASS per step instead of 5). */
#define GG_R2P_MOD_STEP(S, PY, PX)                                                            \
    "shl.b32 ct, %3, " S ";\n\tshr.b32 c, ct, 30;\n\tadd.u32 s, %0, %1;\n\tadd.u32 u, s, c;\n\t"  \
    "selp.b32 o, %0, %1, " PY ";\n\tadd.u32 v, u, o;\n\t"                                   \
    "setp.ge.u32 q, v, %5;\n\t@q sub.u32 v, v, %5;\n\tsetp.ge.u32 q, v, %4;\n\t@q sub.u32 v, v, %4;\n\t" \
    "@" PY " mov.u32 %1, v;\n\t@" PX " mov.u32 %0, v;\n\t"

template <int B0, int B1, int SH0, int SH1>
__device__ __forceinline__ void gg_r2p_two_mod(uint32_t S, uint32_t C, uint32_t m, uint32_t m2,
                                               uint32_t &x, uint32_t &y)
{
    asm volatile(
        "{\n\t.reg .pred py0, px0, py1, px1, q;\n\t.reg .b32 t, ct, c, u, s, o, v;\n\t"
        "and.b32 t, %2, %6;\n\tsetp.ne.b32 py0, t, 0;\n\t"
        "and.b32 t, %2, %7;\n\tsetp.ne.b32 px0, t, 0;\n\t"
        "and.b32 t, %2, %8;\n\tsetp.ne.b32 py1, t, 0;\n\t"
        "and.b32 t, %2, %9;\n\tsetp.ne.b32 px1, t, 0;\n\t"
        GG_R2P_MOD_STEP("%10", "py0", "px0") GG_R2P_MOD_STEP("%11", "py1", "px1") "}"
        : "+r"(x), "+r"(y)
        : "r"(S), "r"(C), "r"(m), "r"(m2), "n"(1u << B0), "n"(2u << B0), "n"(1u << B1),
          "n"(2u << B1), "n"(SH0), "n"(SH1));
}

template <int NK>
__device__ __forceinline__ void gg_word10_r2p_mod(uint32_t Q, uint32_t m, uint32_t m2, uint32_t &x,
                                                  uint32_t &y)
{
    uint32_t C, F;
    gg_r2p_prep(Q, C, F);
    const uint32_t G = F >> 4;
    gg_r2p_two_mod<0, 3, GG_SH(0), GG_SH(1)>(F, C, m, m2, x, y);
    gg_r2p_two_mod<2, 5, GG_SH(2), GG_SH(3)>(G, C, m, m2, x, y);
    if (NK == 4) return;
    gg_r2p_two_mod<8, 11, GG_SH(4), GG_SH(5)>(G, C, m, m2, x, y);
    gg_r2p_two_mod<18, 21, GG_SH(6), GG_SH(7)>(F, C, m, m2, x, y);
    gg_r2p_two_mod<24, 27, GG_SH(8), GG_SH(9)>(F, C, m, m2, x, y);
}

/* 64 steps, forward maps, any m <= 2^30 (x, y < m). */
__device__ __forceinline__ void gg_walk64_r2p_mod(const uint32_t w[6], uint32_t m, uint32_t &x,
                                                  uint32_t &y)
{
    const uint32_t m2 = 2u * m;
    gg_word10_r2p_mod<10>(w[0], m, m2, x, y);
    gg_word10_r2p_mod<10>(__funnelshift_r(w[0], w[1], 30), m, m2, x, y);
    gg_word10_r2p_mod<10>(__funnelshift_r(w[1], w[2], 28), m, m2, x, y);
    gg_word10_r2p_mod<10>(__funnelshift_r(w[2], w[3], 26), m, m2, x, y);
    gg_word10_r2p_mod<10>(__funnelshift_r(w[3], w[4], 24), m, m2, x, y);
    gg_word10_r2p_mod<10>(__funnelshift_r(w[4], w[5], 22), m, m2, x, y);
    gg_word10_r2p_mod<4>(w[5] >> 20, m, m2, x, y);
}

/* One step of the R2P form alone (the first of a pair, flags at bit B0). */
template <int B0, int SH0>
__device__ __forceinline__ void gg_r2p_single(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y)
{
    asm volatile(
        "{\n\t.reg .pred py0, px0;\n\t.reg .b32 t, ct, c, u, s;\n\t"
        "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
        "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
        GG_R2P_U("%6") "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t}"
        : "+r"(x), "+r"(y)
        : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(SH0));
}

/* The first NK (1..10) steps of a 10-field word, forward maps, m = 2^k: the
 * pairs of gg_word10_r2p, the last one cut to its first step for odd NK. */
template <int NK>
__device__ __forceinline__ void gg_word_r2p_n(uint32_t Q, uint32_t &x, uint32_t &y)
{
    uint32_t C, F;
    gg_r2p_prep(Q, C, F);
    const uint32_t G = F >> 4;
    if (NK >= 2) gg_r2p_pair<false, 0, 3, 0>(F, C, x, y);
    else gg_r2p_single<0, GG_SH(0)>(F, C, x, y);
    if (NK >= 4) gg_r2p_pair<false, 2, 5, 2>(G, C, x, y);
    else if (NK == 3) gg_r2p_single<2, GG_SH(2)>(G, C, x, y);
    if (NK >= 6) gg_r2p_pair<false, 8, 11, 4>(G, C, x, y);
    else if (NK == 5) gg_r2p_single<8, GG_SH(4)>(G, C, x, y);
    if (NK >= 8) gg_r2p_pair<false, 18, 21, 6>(F, C, x, y);
    else if (NK == 7) gg_r2p_single<18, GG_SH(6)>(F, C, x, y);
    if (NK >= 10) gg_r2p_pair<false, 24, 27, 8>(F, C, x, y);
    else if (NK == 9) gg_r2p_single<24, GG_SH(8)>(F, C, x, y);
}

/* l steps (any l >= 1), forward maps, m = 2^k, from a record of ceil(3l/32)
 * words at rec[r * stride]: 10-field groups are funnel-shifted out of the
 * record (each word is loaded once) and walked with the R2P step. */
__device__ __forceinline__ void gg_walk_r2p_any(const uint32_t *rec, uint64_t stride, uint32_t l,
                                                uint32_t R, uint32_t &x, uint32_t &y)
{
    uint32_t lo = __ldg(rec), hi = R > 1 ? __ldg(rec + stride) : 0u;
    uint32_t wi = 0;  /* lo = word wi, hi = word wi + 1 (0 past the record) */
    for (uint32_t g = 0; 10u * g < l; g++) {
        const uint32_t bit = 30u * g, i = bit >> 5, sh = bit & 31u;
        if (i != wi) {  /* advance one word (30-bit groups move at most one word) */
            lo = hi;
            wi = i;
            hi = wi + 1 < R ? __ldg(rec + (uint64_t)(wi + 1) * stride) : 0u;
        }
        const uint32_t Q = __funnelshift_r(lo, hi, sh);
        const uint32_t nk = min(10u, l - 10u * g);
        switch (nk) {
        case 10: gg_word_r2p_n<10>(Q, x, y); break;
        case 9: gg_word_r2p_n<9>(Q, x, y); break;
        case 8: gg_word_r2p_n<8>(Q, x, y); break;
        case 7: gg_word_r2p_n<7>(Q, x, y); break;
        case 6: gg_word_r2p_n<6>(Q, x, y); break;
        case 5: gg_word_r2p_n<5>(Q, x, y); break;
        case 4: gg_word_r2p_n<4>(Q, x, y); break;
        case 3: gg_word_r2p_n<3>(Q, x, y); break;
        case 2: gg_word_r2p_n<2>(Q, x, y); break;
        default: gg_word_r2p_n<1>(Q, x, y); break;
        }
    }
}

/* 64 steps from a 6-word record (R2P form).  BIP: the bipartite variant with
 * an even first global step (steps 2i apply sigma, steps 2i+1 sigma^{-1}; every
 * R2P pair is (even, odd) because 10-field words and pairs start at even
 * field indices). */
template <bool BIP = false>
__device__ __forceinline__ void gg_walk64_r2p(const uint32_t w[6], uint32_t &x, uint32_t &y)
{
    gg_word10_r2p<10, BIP>(w[0], x, y);
    gg_word10_r2p<10, BIP>(__funnelshift_r(w[0], w[1], 30), x, y);
    gg_word10_r2p<10, BIP>(__funnelshift_r(w[1], w[2], 28), x, y);
    gg_word10_r2p<10, BIP>(__funnelshift_r(w[2], w[3], 26), x, y);
    gg_word10_r2p<10, BIP>(__funnelshift_r(w[3], w[4], 24), x, y);
    gg_word10_r2p<10, BIP>(__funnelshift_r(w[4], w[5], 22), x, y);
    gg_word10_r2p<4, BIP>(w[5] >> 20, x, y);
}

template <bool BIP = false>
__device__ __forceinline__ void gg_walk64x2_r2p(const uint32_t a[6], const uint32_t b[6], uint32_t &xa,
                                                uint32_t &ya, uint32_t &xb, uint32_t &yb)
{
    gg_word10x2_r2p<10, BIP>(a[0], b[0], xa, ya, xb, yb);
    gg_word10x2_r2p<10, BIP>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb);
    gg_word10x2_r2p<10, BIP>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb);
    gg_word10x2_r2p<10, BIP>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb);
    gg_word10x2_r2p<10, BIP>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb);
    gg_word10x2_r2p<10, BIP>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb);
    gg_word10x2_r2p<4, BIP>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb);
}

/* ------------------------------------------------------------------------
 * Composed-step ("table") walk for l = 64, m = 2^k, forward maps.  The 64
 * steps of a draw are 16 groups of 4 steps (12 record bits each, R3); the
 * composition of a group's 4 steps is one affine map over Z/2^32,
 *     x' = a x + b y + e,  y' = c x + d y + f,
 * with a, d <= 29, b, c <= 22, e, f <= 40 for all 4096 bit patterns, packed
 * a | b<<5 | c<<10 | d<<15 | e<<20 | f<<26 into one 32-bit word.  The
 * library builds the 4096-word table once per device (prng_view::tab); a
 * kernel stages it in shared memory (prng_table_stage) and walks with one
 * lookup and four IMAD per 4 steps (the bulk fill: 311 SASS per number
 * instead of 454 for the R2P step).  Exact: the same wrapped arithmetic as
 * the step-by-step walk, checked in tests/test_table_formulation.py.
 * ------------------------------------------------------------------------ */
#define PRNG_TABLE_WORDS 4096

/* Shared-space address of group G's entry: base + its 12 record bits times
 * 4.  The base is warp-uniform, so ptxas folds the add into the LDS address
 * ([R + UR]).  (An OR with a 16 KB-aligned base is not portable: the CTA's
 * shared window begins with a reserved 1 KB, and ptxas does not honour
 * larger alignments of __shared__ variables.) */
#define PRNG_TABLE_ALIGN 16
template <int G, bool ORB = false>
__device__ __forceinline__ uint32_t prng_group_off(const uint32_t (&w)[6], uint32_t base) {
    constexpr int bit = 12 * G, wi = bit >> 5, sh = bit & 31;
    uint32_t v;
    if constexpr (sh == 0) v = w[wi] << 2;
    else if constexpr (sh <= 20) v = w[wi] >> (sh - 2);
    else v = __funnelshift_r(w[wi], w[wi + 1], sh - 2);
    /* ORB: base is a multiple of 16 KB (library kernels that place the table
     * so), and the OR folds into the masking LOP3 */
    return ORB ? ((v & 0x3FFCu) | base) : ((v & 0x3FFCu) + base);
}

// Left shifts by multiplications with opaque powers of two (IMAD on the
// FMA-heavy pipe), right shifts and masks on the ALU pipe: ptxas would
// otherwise fuse each (t << s) >> r into SHF + LOP3 and put the whole unpack
// on the ALU pipe.
struct prng_tab_shifts {
    uint32_t k22, k17, k12, k6;
};
__device__ __forceinline__ prng_tab_shifts prng_tab_shifts_load() {
    prng_tab_shifts k{1u << 22, 1u << 17, 1u << 12, 1u << 6};
    asm volatile("" : "+r"(k.k22), "+r"(k.k17), "+r"(k.k12), "+r"(k.k6));
    return k;
}

/* SIGNED: the bipartite table's two's-complement fields (arithmetic shifts). */
template <bool SIGNED = false>
__device__ __forceinline__ void prng_group_apply(uint32_t addr, uint32_t &x, uint32_t &y,
                                                 const prng_tab_shifts &k) {
    uint32_t t;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(t) : "r"(addr) : "memory");
    uint32_t a, b, c, d, e, f;
    if (SIGNED) {
        a = (uint32_t)((int32_t)(t << 27) >> 27);
        b = (uint32_t)((int32_t)(t * k.k22) >> 27);
        c = (uint32_t)((int32_t)(t * k.k17) >> 27);
        d = (uint32_t)((int32_t)(t * k.k12) >> 27);
        e = (uint32_t)((int32_t)(t * k.k6) >> 26);
        f = (uint32_t)((int32_t)t >> 26);
    } else {
        a = t & 31u, b = (t * k.k22) >> 27, c = (t * k.k17) >> 27, d = (t * k.k12) >> 27;
        e = (t * k.k6) >> 26, f = t >> 26;
    }
    const uint32_t nx = b * y + (a * x + e);
    const uint32_t ny = d * y + (c * x + f);
    x = nx;
    y = ny;
}

/* Shared-space address (32-bit) of the staged table. */
__device__ __forceinline__ uint32_t prng_table_base(const uint32_t *smem_tab) {
    return (uint32_t)__cvta_generic_to_shared(smem_tab);
}

/* Two walkers, table at shared-space address `base`. */
template <bool SIGNED = false, bool ORB = false>
__device__ __forceinline__ void prng_walk64x2_table_at(uint32_t base, const uint32_t (&wa)[6],
                                                       const uint32_t (&wb)[6], uint32_t &xa,
                                                       uint32_t &ya, uint32_t &xb, uint32_t &yb,
                                                       const prng_tab_shifts &k) {
#define PRNG_TG(G)                                                                \
    prng_group_apply<SIGNED>(prng_group_off<G, ORB>(wa, base), xa, ya, k);        \
    prng_group_apply<SIGNED>(prng_group_off<G, ORB>(wb, base), xb, yb, k);
    PRNG_TG(0) PRNG_TG(1) PRNG_TG(2) PRNG_TG(3) PRNG_TG(4) PRNG_TG(5) PRNG_TG(6) PRNG_TG(7)
    PRNG_TG(8) PRNG_TG(9) PRNG_TG(10) PRNG_TG(11) PRNG_TG(12) PRNG_TG(13) PRNG_TG(14) PRNG_TG(15)
#undef PRNG_TG
}

template <bool SIGNED = false>
__device__ __forceinline__ void prng_walk64x2_table(const uint32_t *tab, const uint32_t (&wa)[6],
                                                  const uint32_t (&wb)[6], uint32_t &xa,
                                                  uint32_t &ya, uint32_t &xb, uint32_t &yb,
                                                  const prng_tab_shifts &k) {
    prng_walk64x2_table_at<SIGNED, false>(prng_table_base(tab), wa, wb, xa, ya, xb, yb, k);
}


__device__ __forceinline__ void prng_walk64_table(const uint32_t *tab, const uint32_t (&w)[6],
                                                  uint32_t &x, uint32_t &y,
                                                  const prng_tab_shifts &k)
{
    const uint32_t base = prng_table_base(tab);
#define PRNG_TG1(G) prng_group_apply(prng_group_off<G>(w, base), x, y, k);
    PRNG_TG1(0) PRNG_TG1(1) PRNG_TG1(2) PRNG_TG1(3) PRNG_TG1(4) PRNG_TG1(5) PRNG_TG1(6) PRNG_TG1(7)
    PRNG_TG1(8) PRNG_TG1(9) PRNG_TG1(10) PRNG_TG1(11) PRNG_TG1(12) PRNG_TG1(13) PRNG_TG1(14) PRNG_TG1(15)
#undef PRNG_TG1
}

/* One step, any m (generic path), x, y < m.  m = 2^k: wrapped 32-bit
 * arithmetic.  Other m <= 2^30: every pre-reduction value is < 4m < 2^32, so
 * two conditional subtracts reduce it.  Other m < 2^32 ("wide"): the same in
 * 64 bits (2x + y + c <= 3m - 1 needs 34 bits).  A multiply-shift (Barrett)
 * reduction is not needed: the quotient is at most 3.
 * inv: apply sigma_k^{-1} (variant 1, odd steps): y - 2x - c / x - 2y - c. */
__device__ __forceinline__ uint32_t gg_reduce(uint32_t t, uint32_t m, bool pow2)
{
    if (!pow2) {
        t = (t >= 2u * m) ? t - 2u * m : t;
        t = (t >= m) ? t - m : t;
    }
    return t;
}

__device__ __forceinline__ uint32_t gg_reduce64(uint64_t t, uint32_t m)  /* t < 4m */
{
    const uint64_t mm = m;
    t = (t >= 2u * mm) ? t - 2u * mm : t;
    t = (t >= mm) ? t - mm : t;
    return (uint32_t)t;
}

__device__ __forceinline__ void gg_step_generic(uint32_t b, uint32_t &x, uint32_t &y,
                                                uint32_t m, bool pow2, bool inv = false)
{
    const uint32_t cy = b - 1u, cx = b - 4u;
    const bool wide = !pow2 && m > (1u << 30);
    if (cy < 3u) {
        if (wide)
            y = inv ? gg_reduce64((uint64_t)y + 3ull * m - 2ull * x - cy, m)
                    : gg_reduce64((uint64_t)y + 2ull * x + cy, m);
        else if (!inv)
            y = gg_reduce(y + 2u * x + cy, m, pow2);
        else
            y = pow2 ? y - 2u * x - cy : gg_reduce(y + 3u * m - 2u * x - cy, m, false);
    } else if (cx < 3u) {
        if (wide)
            x = inv ? gg_reduce64((uint64_t)x + 3ull * m - 2ull * y - cx, m)
                    : gg_reduce64((uint64_t)x + 2ull * y + cx, m);
        else if (!inv)
            x = gg_reduce(x + 2u * y + cx, m, pow2);
        else
            x = pow2 ? x - 2u * y - cx : gg_reduce(x + 3u * m - 2u * y - cx, m, false);
    }
}

/* Field i of a record stored at rec[r*stride] (R3: little-endian bit string). */
__device__ __forceinline__ uint32_t gg_field(const uint32_t *rec, uint64_t stride, uint32_t i)
{
    const uint32_t bit = 3u * i, r = bit >> 5, s = bit & 31u;
    uint32_t lo = rec[(uint64_t)r * stride];
    if (s <= 29u)
        return (lo >> s) & 7u;
    uint32_t hi = rec[(uint64_t)(r + 1) * stride];
    return __funnelshift_r(lo, hi, s) & 7u;
}

/* nsteps steps reading the record from global memory (generic l / m /
 * variant); s0 = global step index of the first step (variant 1 parity). */
__device__ __forceinline__ void gg_walk_generic(const uint32_t *rec, uint64_t stride,
                                                uint32_t nsteps, uint32_t &x, uint32_t &y,
                                                uint32_t m, bool pow2, uint32_t variant = 0,
                                                uint64_t s0 = 0)
{
    for (uint32_t i = 0; i < nsteps; i++)
        gg_step_generic(gg_field(rec, stride, i), x, y, m, pow2,
                        variant == 1 && ((s0 + i) & 1) != 0);
}

/* Vertex label x + m*y (R8), reducing wrapped coordinates for m = 2^k. */
__device__ __forceinline__ uint64_t gg_label(uint32_t x, uint32_t y, uint64_t m, uint32_t log2m,
                                             bool pow2)
{
    if (pow2) {
        const uint32_t mask = (log2m >= 32) ? 0xFFFFFFFFu : ((1u << log2m) - 1u);
        return ((uint64_t)(y & mask) << log2m) | (uint64_t)(x & mask);
    }
    return (uint64_t)x + m * (uint64_t)y;
}

/* ------------------------------ on-demand API -------------------------- */

/* State of the walker in window slot `slot` (= the walker itself unless the
 * epoch was opened with an explicit walker list). */
__device__ __forceinline__ prng_state prng_state_load(const prng_view *v, uint32_t slot)
{
    prng_state st;
    const uint32_t walker = v->wmap ? v->wmap[slot] : slot;
    st.x = v->x[walker];
    st.y = v->y[walker];
    st.walker = walker;
    st.slot = slot;
    st.view = v;
    const uint32_t j = v->j[walker];
    st.used = (j > v->J0) ? (j - v->J0) : 0u; /* walkers that skipped epochs jump to J0 */
    return st;
}

__device__ __forceinline__ void prng_state_store(const prng_view *v, const prng_state *st)
{
    v->x[st->walker] = st->x;
    v->y[st->walker] = st->y;
    v->j[st->walker] = v->J0 + st->used;
}

/* Draws left in the current window for this walker. */
__device__ __forceinline__ uint32_t prng_available(const prng_view *v, const prng_state *st)
{
    return (st->used < v->D) ? (v->D - st->used) : 0u;
}

/* One-argument forms: the state carries its view. */
__device__ __forceinline__ uint32_t prng_available(const prng_state *st)
{
    return prng_available(st->view, st);
}

__device__ __forceinline__ void prng_state_store(const prng_state *st)
{
    prng_state_store(st->view, st);
}

/* Walk implementations prng_next can use, picked from the view's (m, l,
 * variant, l0).  A kernel that knows its generator's shape instantiates
 * prng_next<MODE> so only that walk is compiled into it; prng_next without a
 * mode (PRNG_WALK_AUTO) dispatches at run time over all of them.  Every mode
 * returns the same numbers as the generic walk for the views it accepts. */
enum {
    PRNG_WALK_AUTO = 0,      /* run-time dispatch (any view) */
    PRNG_WALK_L64 = 1,       /* l = 64, m = 2^k, forward maps (the paper's generator) */
    PRNG_WALK_L64_BIP = 2,   /* l = 64, m = 2^k, bipartite, l0 even (draws start at even steps) */
    PRNG_WALK_ANY_POW2 = 3,  /* any l, m = 2^k, forward maps */
    PRNG_WALK_L64_MOD = 4,   /* l = 64, m <= 2^30 not a power of two, forward maps */
    PRNG_WALK_GENERIC = 5    /* anything (per-step field loads, conditional-subtract mod m) */
};

/* The fastest mode that is exact for this view (host or device). */
static inline __host__ __device__ int prng_walk_mode(const prng_view *v)
{
    if (v->l == 64u && v->pow2 && v->variant == 0) return PRNG_WALK_L64;
    if (v->l == 64u && v->pow2 && v->variant == 1 && (v->l0 & 1u) == 0) return PRNG_WALK_L64_BIP;
    if (v->pow2 && v->variant == 0) return PRNG_WALK_ANY_POW2;
    if (v->l == 64u && v->variant == 0 && v->m <= (1ull << 30)) return PRNG_WALK_L64_MOD;
    return PRNG_WALK_GENERIC;
}

/* One walk of l steps from (x, y) with the record at rec (column stride
 * pitch), in walk mode MODE (not AUTO). */
template <int MODE>
__device__ __forceinline__ void prng_walk_mode_apply(const prng_view *v, const uint32_t *rec,
                                                     uint32_t draw_in_window, uint32_t &x,
                                                     uint32_t &y)
{
    if (MODE == PRNG_WALK_L64 || MODE == PRNG_WALK_L64_BIP || MODE == PRNG_WALK_L64_MOD) {
        uint32_t w[6];
#pragma unroll
        for (int r = 0; r < 6; r++)
            w[r] = __ldg(rec + (uint64_t)r * v->pitch);
        if (MODE == PRNG_WALK_L64)
            gg_walk64_r2p(w, x, y);
        else if (MODE == PRNG_WALK_L64_BIP)
            gg_walk64_r2p<true>(w, x, y);  /* draw starts at global step l0 + 64 j: even */
        else
            gg_walk64_r2p_mod(w, (uint32_t)v->m, x, y);
    } else if (MODE == PRNG_WALK_ANY_POW2) {
        gg_walk_r2p_any(rec, v->pitch, v->l, v->R, x, y);
    } else {
        const uint64_t s0 = (uint64_t)v->l0 + (uint64_t)v->l * (v->J0 + draw_in_window);
        gg_walk_generic(rec, v->pitch, v->l, x, y, (uint32_t)v->m, v->pow2 != 0, v->variant, s0);
    }
}

/* Alg.2 GetNextRand: walk l steps with the bits of draw (J0 + used).
 * MODE = PRNG_WALK_AUTO picks the walk at run time; a fixed MODE must be
 * prng_walk_mode(v) (or PRNG_WALK_GENERIC, which accepts any view). */
template <int MODE = PRNG_WALK_AUTO>
__device__ __forceinline__ uint64_t prng_next(prng_state *st, const prng_view *v)
{
    if (st->used >= v->D || st->slot >= v->Wv) {
        atomicOr(v->flags, PRNG_FLAG_OVERRUN);
        return 0ull;
    }
    const uint32_t *rec = v->bits + (uint64_t)st->used * v->R * v->pitch + st->slot;
    uint32_t x = st->x, y = st->y;
    if (MODE == PRNG_WALK_AUTO) {
        switch (prng_walk_mode(v)) {
        case PRNG_WALK_L64: prng_walk_mode_apply<PRNG_WALK_L64>(v, rec, st->used, x, y); break;
        case PRNG_WALK_L64_BIP:
            prng_walk_mode_apply<PRNG_WALK_L64_BIP>(v, rec, st->used, x, y);
            break;
        case PRNG_WALK_ANY_POW2:
            prng_walk_mode_apply<PRNG_WALK_ANY_POW2>(v, rec, st->used, x, y);
            break;
        case PRNG_WALK_L64_MOD:
            prng_walk_mode_apply<PRNG_WALK_L64_MOD>(v, rec, st->used, x, y);
            break;
        default: prng_walk_mode_apply<PRNG_WALK_GENERIC>(v, rec, st->used, x, y); break;
        }
    } else {
        prng_walk_mode_apply<MODE>(v, rec, st->used, x, y);
    }
    st->x = x;
    st->y = y;
    st->used++;
    const bool pow2 = (MODE == PRNG_WALK_L64 || MODE == PRNG_WALK_L64_BIP ||
                       MODE == PRNG_WALK_ANY_POW2) ? true
                      : (MODE == PRNG_WALK_L64_MOD) ? false : (v->pow2 != 0);
    return gg_label(x, y, v->m, v->log2m, pow2);
}

/* north_star's one-argument form prng_next(&state): the state remembers the
 * view it was loaded from (prng_state_load).  Same numbers as
 * prng_next(&state, view). */
template <int MODE = PRNG_WALK_AUTO>
__device__ __forceinline__ uint64_t prng_next(prng_state *st)
{
    return prng_next<MODE>(st, st->view);
}

/* K draws at once: the K records' loads are issued together before the
 * first walk, so a consumer that needs several numbers per iteration (the
 * Monte Carlo consumer takes three) waits for memory once, not K times.
 * Same numbers, same order, same overrun rule as K calls of prng_next.
 * The batched form needs l = 64, m = 2^k, forward maps (MODE L64, or AUTO
 * on such a view); every other view takes K single calls. */
template <int K, bool ROLL = false, int MODE = PRNG_WALK_AUTO>
__device__ __forceinline__ void prng_next_n(prng_state *st, const prng_view *v, uint64_t (&out)[K])
{
    const bool l64 = MODE == PRNG_WALK_L64 ||
                     (MODE == PRNG_WALK_AUTO && prng_walk_mode(v) == PRNG_WALK_L64);
    if (!l64 || st->used + K > v->D || st->slot >= v->Wv) {
#pragma unroll
        for (int k = 0; k < K; k++) out[k] = prng_next<MODE>(st, v);
        return;
    }
    uint32_t w[K][6];
#pragma unroll
    for (int k = 0; k < K; k++) {
        const uint32_t *rec = v->bits + (uint64_t)(st->used + k) * 6u * v->pitch + st->slot;
#pragma unroll
        for (int r = 0; r < 6; r++) w[k][r] = __ldg(rec + (uint64_t)r * v->pitch);
    }
    uint32_t x = st->x, y = st->y;
    if (!ROLL) {
#pragma unroll
        for (int k = 0; k < K; k++) {
            gg_walk64_r2p(w[k], x, y);
            out[k] = gg_label(x, y, v->m, v->log2m, true);
        }
        st->x = x;
        st->y = y;
        st->used += K;
        return;
    }
    /* ROLL: one copy of the walk in a rolled loop (the records rotate through
     * w[0] with register moves), for consumers whose hot loop would not fit
     * the instruction cache with K unrolled walks (Monte Carlo: ncu "no
     * instruction" stalls; 28.5 -> 30.9 G draws/s in-kernel).  Kernels with a
     * small body keep the unrolled form (gg_consume: 65.7 vs 61.2 G/s rolled). */
#pragma unroll 1
    for (int k = 0; k < K; k++) {
        gg_walk64_r2p(w[0], x, y);
        uint64_t lab = gg_label(x, y, v->m, v->log2m, true);
#pragma unroll
        for (int q = 0; q < K; q++)
            if (q == k) out[q] = lab;
#pragma unroll
        for (int q = 0; q + 1 < K; q++)
#pragma unroll
            for (int r = 0; r < 6; r++) w[q][r] = w[q + 1][r];
    }
    st->x = x;
    st->y = y;
    st->used += K;
}

/* ---------------- on demand with the composed-step table ----------------
 * For views with prng_walk_mode(v) == PRNG_WALK_L64 (the paper's generator):
 *     __shared__ __align__(PRNG_TABLE_ALIGN) uint32_t tab[PRNG_TABLE_WORDS];  // 16 KB
 *     prng_table_stage(&view, tab);  __syncthreads();   // every thread of the block
 *     ... uint64_t r = prng_next_table(&st, &view, tab);
 * Same numbers as prng_next; other views ignore the table (prng_next). */
__device__ __forceinline__ void prng_table_stage(const prng_view *v, uint32_t *smem_tab)
{
    const uint4 *src = reinterpret_cast<const uint4 *>(v->tab);
    uint4 *dst = reinterpret_cast<uint4 *>(smem_tab);
    const uint32_t nthreads = blockDim.x * blockDim.y * blockDim.z;
    const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
    for (uint32_t i = tid; i < PRNG_TABLE_WORDS / 4; i += nthreads) dst[i] = __ldg(src + i);
}

__device__ __forceinline__ uint64_t prng_next_table(prng_state *st, const prng_view *v,
                                                    const uint32_t *smem_tab)
{
    if (prng_walk_mode(v) != PRNG_WALK_L64) return prng_next(st, v);
    if (st->used >= v->D || st->slot >= v->Wv) {
        atomicOr(v->flags, PRNG_FLAG_OVERRUN);
        return 0ull;
    }
    const uint32_t *rec = v->bits + (uint64_t)st->used * 6u * v->pitch + st->slot;
    uint32_t w[6];
#pragma unroll
    for (int r = 0; r < 6; r++) w[r] = __ldg(rec + (uint64_t)r * v->pitch);
    uint32_t x = st->x, y = st->y;
    prng_walk64_table(smem_tab, w, x, y, prng_tab_shifts_load());
    st->x = x;
    st->y = y;
    st->used++;
    return gg_label(x, y, v->m, v->log2m, true);
}

/* K draws with the table, records loaded together (prng_next_n's contract);
 * ROLL: one walk copy in a rolled loop. */
template <int K, bool ROLL = false>
__device__ __forceinline__ void prng_next_n_table(prng_state *st, const prng_view *v,
                                                  const uint32_t *smem_tab, uint64_t (&out)[K])
{
    if (prng_walk_mode(v) != PRNG_WALK_L64 || st->used + K > v->D || st->slot >= v->Wv) {
#pragma unroll
        for (int k = 0; k < K; k++) out[k] = prng_next_table(st, v, smem_tab);
        return;
    }
    uint32_t w[K][6];
#pragma unroll
    for (int k = 0; k < K; k++) {
        const uint32_t *rec = v->bits + (uint64_t)(st->used + k) * 6u * v->pitch + st->slot;
#pragma unroll
        for (int r = 0; r < 6; r++) w[k][r] = __ldg(rec + (uint64_t)r * v->pitch);
    }
    const prng_tab_shifts ks = prng_tab_shifts_load();
    uint32_t x = st->x, y = st->y;
    if (!ROLL) {
#pragma unroll
        for (int k = 0; k < K; k++) {
            prng_walk64_table(smem_tab, w[k], x, y, ks);
            out[k] = gg_label(x, y, v->m, v->log2m, true);
        }
    } else {
#pragma unroll 1
        for (int k = 0; k < K; k++) {
            prng_walk64_table(smem_tab, w[0], x, y, ks);
            const uint64_t lab = gg_label(x, y, v->m, v->log2m, true);
#pragma unroll
            for (int q = 0; q < K; q++)
                if (q == k) out[q] = lab;
#pragma unroll
            for (int q = 0; q + 1 < K; q++)
#pragma unroll
                for (int r = 0; r < 6; r++) w[q][r] = w[q + 1][r];
        }
    }
    st->x = x;
    st->y = y;
    st->used += K;
}

#endif /* GGPRNG_PRNG_DEVICE_CUH */
