// Step-formulation microbenchmark on sm_100a (tool, not product): each variant runs the
// l = 64 walk (two walkers per thread, records read by LDG) and must agree bit-exactly with V6
// (the product step).  Run under ncu with sm__inst_executed_pipe_{alu,fmaheavy,fmalite} to see
// how each formulation loads the ALU and FMA-heavy pipes.
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <vector>
#include <cuda_runtime.h>

// V6: product step  u = x + y + c ; y' = u + x | x' = u + y
// VH: h = hi(ct*4) + y (IMAD.HI) ; y' = 2x + h | x' = x + y + h
// VL: h = y + (ct >> 30) (LEA.HI) ; y' = 2x + h | x' = x + y + h
// VM: h via LEA.HI, s = x + y, x' = s + h
template <int V, int K>
__device__ __forceinline__ void step(uint32_t MY, uint32_t MX, uint32_t C, uint32_t &x, uint32_t &y, uint32_t four) {
  if (V == 6) {
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, u, s;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shl.b32 ct, %4, %6;\n\tshr.b32 c, ct, 30;\n\tadd.u32 s, %0, %1;\n\tadd.u32 u, s, c;\n\t"
      "@py add.u32 %1, u, %0;\n\t@px add.u32 %0, u, %1;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K));
  } else if (V == 1) {
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, h, s;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shl.b32 ct, %4, %6;\n\tmad.hi.u32 h, ct, %7, %1;\n\tadd.u32 s, %0, %1;\n\t"
      "@py mad.lo.u32 %1, %0, 2, h;\n\t@px add.u32 %0, s, h;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "r"(four));
  } else if (V == 2) {
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, h, s;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shl.b32 ct, %4, %6;\n\tshr.b32 c, ct, 30;\n\tadd.u32 h, %1, c;\n\tadd.u32 s, %0, %1;\n\t"
      "@py mad.lo.u32 %1, %0, 2, h;\n\t@px add.u32 %0, s, h;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K));
  } else {  // V3: y' via shl-add (LEA, ALU) instead of IMAD
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, h, s, x2;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "mul.lo.u32 ct, %4, %7;\n\tmad.hi.u32 h, ct, %8, %1;\n\tadd.u32 s, %0, %1;\n\t"
      "@py mad.lo.u32 %1, %0, 2, h;\n\t@px add.u32 %0, s, h;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "n"(1u << (30 - 3*K)), "r"(four));
  }
}
template <int V, int NK>
__device__ __forceinline__ void word10x2(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                         uint32_t &xb, uint32_t &yb, uint32_t four) {
  const uint32_t f1a = Qa >> 1, f2a = Qa >> 2, f1b = Qb >> 1, f2b = Qb >> 2;
  const uint32_t MYa = ~f2a & (f1a | Qa), MXa = f2a & ~(f1a & Qa), Ca = Qa - (MYa & 0x09249249u);
  const uint32_t MYb = ~f2b & (f1b | Qb), MXb = f2b & ~(f1b & Qb), Cb = Qb - (MYb & 0x09249249u);
#define S2(k) if (NK > k) { step<V, k>(MYa, MXa, Ca, xa, ya, four); step<V, k>(MYb, MXb, Cb, xb, yb, four); }
  S2(0) S2(1) S2(2) S2(3) S2(4) S2(5) S2(6) S2(7) S2(8) S2(9)
#undef S2
}

// V10: IMAD.WIDE chain.  Per 10-field word: C = brev(fields laid out (0, c1, c0)) so that
// {C', c} = C * 8 yields the step constant c in the high word; MY / MX flags at field bits 1 / 2.
template <int K>
__device__ __forceinline__ void stepW(uint32_t &C, uint32_t MY, uint32_t MX, uint32_t &x, uint32_t &y, uint32_t eight) {
  asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b64 d;\n\t.reg .b32 t, c, u;\n\t"
    "mul.wide.u32 d, %2, %5;\n\t"
    "mov.b64 {%2, c}, d;\n\t"
    "and.b32 t, %3, %6;\n\tsetp.ne.b32 py, t, 0;\n\t"
    "and.b32 t, %4, %7;\n\tsetp.ne.b32 px, t, 0;\n\t"
    "add.u32 u, %0, %1;\n\tadd.u32 u, u, c;\n\t"
    "@py add.u32 %1, u, %0;\n\t"
    "@px add.u32 %0, u, %1;\n\t}"
    : "+r"(x), "+r"(y), "+r"(C) : "r"(MY), "r"(MX), "r"(eight), "n"(2u << (3*K)), "n"(4u << (3*K)));
}
__device__ __forceinline__ void prepW(uint32_t Q, uint32_t &C, uint32_t &MY, uint32_t &MX) {
  const uint32_t q1l = Q << 1, q2l = Q << 2, q1r = Q >> 1;
  MY = (Q | q1l) & ~q1r;
  MX = Q & ~(q1l & q2l);
  const uint32_t c1 = (Q & 0x12492492u) & (q1l ^ q1r);
  const uint32_t c0 = (q2l ^ q1l) & (q1l ^ Q);
  C = __brev(c1 | (c0 & 0x24924924u));
}
template <int NK>
__device__ __forceinline__ void word10x2W(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                          uint32_t &xb, uint32_t &yb, uint32_t eight) {
  uint32_t Ca, MYa, MXa, Cb, MYb, MXb;
  prepW(Qa, Ca, MYa, MXa); prepW(Qb, Cb, MYb, MXb);
#define S2(k) if (NK > k) { stepW<k>(Ca, MYa, MXa, xa, ya, eight); stepW<k>(Cb, MYb, MXb, xb, yb, eight); }
  S2(0) S2(1) S2(2) S2(3) S2(4) S2(5) S2(6) S2(7) S2(8) S2(9)
#undef S2
}

// V11: IMAD.WIDE chain + R2P.  F holds py at field bit 1 and px at field bit 2 (F = MY@1 | MX@2);
// G = F >> 6.  Each asm block does two steps whose four flags sit in one byte of F or G, so
// ptxas loads them with a single R2P (bytes hold at most 7 usable bits).
template <int B0, int B1>   // bit positions (in src) of step-0 py and step-1 py; px = py + 1
__device__ __forceinline__ void two11(uint32_t S, uint32_t &C, uint32_t &x, uint32_t &y, uint32_t eight) {
  asm volatile("{\n\t.reg .pred py0, px0, py1, px1;\n\t.reg .b64 d;\n\t.reg .b32 t, c, u;\n\t"
    "and.b32 t, %3, %5;\n\tsetp.ne.b32 py0, t, 0;\n\t"
    "and.b32 t, %3, %6;\n\tsetp.ne.b32 px0, t, 0;\n\t"
    "and.b32 t, %3, %7;\n\tsetp.ne.b32 py1, t, 0;\n\t"
    "and.b32 t, %3, %8;\n\tsetp.ne.b32 px1, t, 0;\n\t"
    "mul.wide.u32 d, %2, %4;\n\tmov.b64 {%2, c}, d;\n\t"
    "add.u32 u, %0, %1;\n\tadd.u32 u, u, c;\n\t"
    "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t"
    "mul.wide.u32 d, %2, %4;\n\tmov.b64 {%2, c}, d;\n\t"
    "add.u32 u, %0, %1;\n\tadd.u32 u, u, c;\n\t"
    "@py1 add.u32 %1, u, %0;\n\t@px1 add.u32 %0, u, %1;\n\t}"
    : "+r"(x), "+r"(y), "+r"(C) : "r"(S), "r"(eight), "n"(1u << B0), "n"(2u << B0), "n"(1u << B1), "n"(2u << B1));
}
template <int B0>
__device__ __forceinline__ void one11(uint32_t S, uint32_t &C, uint32_t &x, uint32_t &y, uint32_t eight) {
  asm volatile("{\n\t.reg .pred py0, px0;\n\t.reg .b64 d;\n\t.reg .b32 t, c, u;\n\t"
    "and.b32 t, %3, %5;\n\tsetp.ne.b32 py0, t, 0;\n\t"
    "and.b32 t, %3, %6;\n\tsetp.ne.b32 px0, t, 0;\n\t"
    "mul.wide.u32 d, %2, %4;\n\tmov.b64 {%2, c}, d;\n\t"
    "add.u32 u, %0, %1;\n\tadd.u32 u, u, c;\n\t"
    "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t}"
    : "+r"(x), "+r"(y), "+r"(C) : "r"(S), "r"(eight), "n"(1u << B0), "n"(2u << B0));
}
__device__ __forceinline__ void prep11(uint32_t Q, uint32_t &C, uint32_t &F) {
  const uint32_t q1l = Q << 1, q2l = Q << 2, q1r = Q >> 1;
  const uint32_t MY = (Q | q1l) & ~q1r;        // py at field bit 1
  const uint32_t MX = Q & ~(q1l & q2l);        // px at field bit 2
  F = (MY & 0x12492492u) | (MX & ~0x12492492u);
  const uint32_t c1 = (Q & 0x12492492u) & (q1l ^ q1r);
  const uint32_t c0 = (q2l ^ q1l) & (q1l ^ Q);
  C = __brev(c1 | (c0 & 0x24924924u));
}
template <int NK>
__device__ __forceinline__ void word10x2R(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                          uint32_t &xb, uint32_t &yb, uint32_t eight) {
  uint32_t Ca, Fa, Cb, Fb;
  prep11(Qa, Ca, Fa); prep11(Qb, Cb, Fb);
  const uint32_t Ga = Fa >> 6, Gb = Fb >> 6;
  two11<1, 4>(Fa, Ca, xa, ya, eight); two11<1, 4>(Fb, Cb, xb, yb, eight);     // steps 0,1: F.B0
  two11<1, 4>(Ga, Ca, xa, ya, eight); two11<1, 4>(Gb, Cb, xb, yb, eight);     // steps 2,3: G.B0
  if (NK > 4) {
    one11<13>(Fa, Ca, xa, ya, eight); one11<13>(Fb, Cb, xb, yb, eight);       // step 4: F.B1
    two11<10, 13>(Ga, Ca, xa, ya, eight); two11<10, 13>(Gb, Cb, xb, yb, eight); // steps 5,6: G.B1
    two11<16, 19>(Ga, Ca, xa, ya, eight); two11<16, 19>(Gb, Cb, xb, yb, eight); // steps 7,8: G.B2
    one11<28>(Fa, Ca, xa, ya, eight); one11<28>(Fb, Cb, xb, yb, eight);       // step 9: F.B3
  }
}

// V12: c by shift + LEA.HI (h = y + c), y' = 2x + h (IMAD), x' = x + y + h (IADD3); predicates by R2P
// from F = MY@3i | MX@3i+1 (and G = F >> 6 for the steps whose flags straddle a byte).
#define STEP12(P, Q, K) \
    "shl.b32 ct, %3, " #K ";\n\tshr.b32 c, ct, 30;\n\tadd.u32 h, %1, c;\n\t" \
    "add.u32 s, %0, %1;\n\t" \
    "@" #P " mad.lo.u32 %1, %0, 2, h;\n\t@" #Q " add.u32 %0, s, h;\n\t"
template <int B0, int B1, int S0, int S1>
__device__ __forceinline__ void two12(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y) {
  asm volatile("{\n\t.reg .pred py0, px0, py1, px1;\n\t.reg .b32 t, ct, c, h, s;\n\t"
    "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
    "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
    "and.b32 t, %2, %6;\n\tsetp.ne.b32 py1, t, 0;\n\t"
    "and.b32 t, %2, %7;\n\tsetp.ne.b32 px1, t, 0;\n\t"
    "shl.b32 ct, %3, %8;\n\tshr.b32 c, ct, 30;\n\tadd.u32 h, %1, c;\n\tadd.u32 s, %0, %1;\n\t"
    "add.u32 t, %0, %0;\n\t@py0 add.u32 %1, t, h;\n\t@px0 add.u32 %0, s, h;\n\t"
    "shl.b32 ct, %3, %9;\n\tshr.b32 c, ct, 30;\n\tadd.u32 h, %1, c;\n\tadd.u32 s, %0, %1;\n\t"
    "add.u32 t, %0, %0;\n\t@py1 add.u32 %1, t, h;\n\t@px1 add.u32 %0, s, h;\n\t}"
    : "+r"(x), "+r"(y) : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(1u << B1), "n"(2u << B1),
      "n"(S0), "n"(S1));
}
template <int B0, int S0>
__device__ __forceinline__ void one12(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y) {
  asm volatile("{\n\t.reg .pred py0, px0;\n\t.reg .b32 t, ct, c, h, s;\n\t"
    "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
    "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
    "shl.b32 ct, %3, %6;\n\tshr.b32 c, ct, 30;\n\tadd.u32 h, %1, c;\n\tadd.u32 s, %0, %1;\n\t"
    "@py0 mad.lo.u32 %1, %0, 2, h;\n\t@px0 add.u32 %0, s, h;\n\t}"
    : "+r"(x), "+r"(y) : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(S0));
}
__device__ __forceinline__ void prep12(uint32_t Q, uint32_t &C, uint32_t &F) {
  const uint32_t f1 = Q >> 1, f2 = Q >> 2;
  const uint32_t MY = ((f1 | Q) & 0x09249249u) & ~f2;
  const uint32_t MX = f2 & ~(f1 & Q);
  C = Q - MY;
  F = MY | ((MX << 1) & 0x12492492u);
}
#define SH(k) (30 - 3 * (k))
template <int NK>
__device__ __forceinline__ void word10x2T(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                          uint32_t &xb, uint32_t &yb) {
  uint32_t Ca, Fa, Cb, Fb;
  prep12(Qa, Ca, Fa); prep12(Qb, Cb, Fb);
  const uint32_t Ga = Fa >> 6, Gb = Fb >> 6;
  two12<0, 3, SH(0), SH(1)>(Fa, Ca, xa, ya); two12<0, 3, SH(0), SH(1)>(Fb, Cb, xb, yb);
  if (NK == 4) {
    two12<0, 3, SH(2), SH(3)>(Ga, Ca, xa, ya); two12<0, 3, SH(2), SH(3)>(Gb, Cb, xb, yb);
    return;
  }
  one12<0, SH(2)>(Ga, Ca, xa, ya); one12<0, SH(2)>(Gb, Cb, xb, yb);
  two12<9, 12, SH(3), SH(4)>(Fa, Ca, xa, ya); two12<9, 12, SH(3), SH(4)>(Fb, Cb, xb, yb);
  one12<9, SH(5)>(Ga, Ca, xa, ya); one12<9, SH(5)>(Gb, Cb, xb, yb);
  two12<18, 21, SH(6), SH(7)>(Fa, Ca, xa, ya); two12<18, 21, SH(6), SH(7)>(Fb, Cb, xb, yb);
  two12<24, 27, SH(8), SH(9)>(Fa, Ca, xa, ya); two12<24, 27, SH(8), SH(9)>(Fb, Cb, xb, yb);
}

// V13: the product step (u = x + y + c by IMAD.SHL + LEA.HI, @py y = u + x, @px x = u + y) with
// predicates loaded by R2P from F = MY@3i | MX@3i+1 (G = F >> 6 for steps 2 and 5).
#define US13(S) "shl.b32 ct, %3, " S ";\n\tshr.b32 c, ct, 30;\n\tadd.u32 s, %0, %1;\n\tadd.u32 u, s, c;\n\t"
template <int B0, int B1, int S0, int S1>
__device__ __forceinline__ void two13(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y) {
  asm volatile("{\n\t.reg .pred py0, px0, py1, px1;\n\t.reg .b32 t, ct, c, u, s;\n\t"
    "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
    "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
    "and.b32 t, %2, %6;\n\tsetp.ne.b32 py1, t, 0;\n\t"
    "and.b32 t, %2, %7;\n\tsetp.ne.b32 px1, t, 0;\n\t"
    US13("%8") "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t"
    US13("%9") "@py1 add.u32 %1, u, %0;\n\t@px1 add.u32 %0, u, %1;\n\t}"
    : "+r"(x), "+r"(y) : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(1u << B1), "n"(2u << B1),
      "n"(S0), "n"(S1));
}
template <int B0, int S0>
__device__ __forceinline__ void one13(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y) {
  asm volatile("{\n\t.reg .pred py0, px0;\n\t.reg .b32 t, ct, c, u, s;\n\t"
    "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
    "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
    US13("%6") "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t}"
    : "+r"(x), "+r"(y) : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(S0));
}
template <int NK>
__device__ __forceinline__ void word10x2U(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                          uint32_t &xb, uint32_t &yb) {
  uint32_t Ca, Fa, Cb, Fb;
  prep12(Qa, Ca, Fa); prep12(Qb, Cb, Fb);
  const uint32_t Ga = Fa >> 6, Gb = Fb >> 6;
  two13<0, 3, SH(0), SH(1)>(Fa, Ca, xa, ya); two13<0, 3, SH(0), SH(1)>(Fb, Cb, xb, yb);
  if (NK == 4) {
    two13<0, 3, SH(2), SH(3)>(Ga, Ca, xa, ya); two13<0, 3, SH(2), SH(3)>(Gb, Cb, xb, yb);
    return;
  }
  one13<0, SH(2)>(Ga, Ca, xa, ya); one13<0, SH(2)>(Gb, Cb, xb, yb);
  two13<9, 12, SH(3), SH(4)>(Fa, Ca, xa, ya); two13<9, 12, SH(3), SH(4)>(Fb, Cb, xb, yb);
  one13<9, SH(5)>(Ga, Ca, xa, ya); one13<9, SH(5)>(Gb, Cb, xb, yb);
  two13<18, 21, SH(6), SH(7)>(Fa, Ca, xa, ya); two13<18, 21, SH(6), SH(7)>(Fb, Cb, xb, yb);
  two13<24, 27, SH(8), SH(9)>(Fa, Ca, xa, ya); two13<24, 27, SH(8), SH(9)>(Fb, Cb, xb, yb);
}
#define US14(S) "shl.b32 ct, %3, " S ";\n\tshr.b32 c, ct, 30;\n\tadd.u32 s, %0, c;\n\tadd.u32 u, s, %1;\n\t"
template <int B0, int B1, int S0, int S1>
__device__ __forceinline__ void two14(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y) {
  asm volatile("{\n\t.reg .pred py0, px0, py1, px1;\n\t.reg .b32 t, ct, c, u, s;\n\t"
    "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
    "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
    "and.b32 t, %2, %6;\n\tsetp.ne.b32 py1, t, 0;\n\t"
    "and.b32 t, %2, %7;\n\tsetp.ne.b32 px1, t, 0;\n\t"
    US14("%8") "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t"
    US14("%9") "@py1 add.u32 %1, u, %0;\n\t@px1 add.u32 %0, u, %1;\n\t}"
    : "+r"(x), "+r"(y) : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(1u << B1), "n"(2u << B1),
      "n"(S0), "n"(S1));
}
template <int B0, int S0>
__device__ __forceinline__ void one14(uint32_t S, uint32_t C, uint32_t &x, uint32_t &y) {
  asm volatile("{\n\t.reg .pred py0, px0;\n\t.reg .b32 t, ct, c, u, s;\n\t"
    "and.b32 t, %2, %4;\n\tsetp.ne.b32 py0, t, 0;\n\t"
    "and.b32 t, %2, %5;\n\tsetp.ne.b32 px0, t, 0;\n\t"
    US14("%6") "@py0 add.u32 %1, u, %0;\n\t@px0 add.u32 %0, u, %1;\n\t}"
    : "+r"(x), "+r"(y) : "r"(S), "r"(C), "n"(1u << B0), "n"(2u << B0), "n"(S0));
}
template <int NK>
__device__ __forceinline__ void word10x2Z(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                          uint32_t &xb, uint32_t &yb) {
  uint32_t Ca, Fa, Cb, Fb;
  prep12(Qa, Ca, Fa); prep12(Qb, Cb, Fb);
  const uint32_t Ga = Fa >> 6, Gb = Fb >> 6;
  two14<0, 3, SH(0), SH(1)>(Fa, Ca, xa, ya); two14<0, 3, SH(0), SH(1)>(Fb, Cb, xb, yb);
  if (NK == 4) {
    two14<0, 3, SH(2), SH(3)>(Ga, Ca, xa, ya); two14<0, 3, SH(2), SH(3)>(Gb, Cb, xb, yb);
    return;
  }
  one14<0, SH(2)>(Ga, Ca, xa, ya); one14<0, SH(2)>(Gb, Cb, xb, yb);
  two14<9, 12, SH(3), SH(4)>(Fa, Ca, xa, ya); two14<9, 12, SH(3), SH(4)>(Fb, Cb, xb, yb);
  one14<9, SH(5)>(Ga, Ca, xa, ya); one14<9, SH(5)>(Gb, Cb, xb, yb);
  two14<18, 21, SH(6), SH(7)>(Fa, Ca, xa, ya); two14<18, 21, SH(6), SH(7)>(Fb, Cb, xb, yb);
  two14<24, 27, SH(8), SH(9)>(Fa, Ca, xa, ya); two14<24, 27, SH(8), SH(9)>(Fb, Cb, xb, yb);
}
template <int V>
__device__ __forceinline__ void walk64x2(const uint32_t a[6], const uint32_t b[6], uint32_t &xa, uint32_t &ya,
                                         uint32_t &xb, uint32_t &yb, uint32_t four) {
  if (V == 13) {
    word10x2U<10>(a[0], b[0], xa, ya, xb, yb);
    word10x2U<10>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb);
    word10x2U<10>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb);
    word10x2U<10>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb);
    word10x2U<10>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb);
    word10x2U<10>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb);
    word10x2U<4>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb);
    return;
  }
  if (V == 14) {
    word10x2Z<10>(a[0], b[0], xa, ya, xb, yb);
    word10x2Z<10>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb);
    word10x2Z<10>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb);
    word10x2Z<10>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb);
    word10x2Z<10>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb);
    word10x2Z<10>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb);
    word10x2Z<4>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb);
    return;
  }
  if (V == 12) {
    word10x2T<10>(a[0], b[0], xa, ya, xb, yb);
    word10x2T<10>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb);
    word10x2T<10>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb);
    word10x2T<10>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb);
    word10x2T<10>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb);
    word10x2T<10>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb);
    word10x2T<4>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb);
    return;
  }
  if (V == 11) {
    const uint32_t e = four * 2u;
    word10x2R<10>(a[0], b[0], xa, ya, xb, yb, e);
    word10x2R<10>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb, e);
    word10x2R<10>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb, e);
    word10x2R<10>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb, e);
    word10x2R<10>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb, e);
    word10x2R<10>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb, e);
    word10x2R<4>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb, e);
    return;
  }
  if (V == 10) {
    const uint32_t e = four * 2u;
    word10x2W<10>(a[0], b[0], xa, ya, xb, yb, e);
    word10x2W<10>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb, e);
    word10x2W<10>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb, e);
    word10x2W<10>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb, e);
    word10x2W<10>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb, e);
    word10x2W<10>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb, e);
    word10x2W<4>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb, e);
    return;
  }
  word10x2<V,10>(a[0], b[0], xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb, four);
  word10x2<V,4>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb, four);
}
template <int V>
__global__ void __launch_bounds__(64) kfill2(const uint32_t* __restrict__ bits, uint64_t pitch, uint32_t W, uint32_t D,
                                             uint32_t* xs, uint32_t* ys, uint64_t* out, uint32_t units, uint32_t four) {
  const uint32_t lane = threadIdx.x & 31u, warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t u = warp; u < units / 2; u += nwarps) {
    const uint32_t ta = u * 64u + lane, tb = ta + 32u;
    uint32_t xa = xs[ta], ya = ys[ta], xb = xs[tb], yb = ys[tb];
    uint32_t a0[6], b0[6], a1[6], b1[6];
#pragma unroll
    for (int r = 0; r < 6; r++) {
      a0[r] = __ldg(bits + ta + (uint64_t)r * pitch); b0[r] = __ldg(bits + tb + (uint64_t)r * pitch);
      a1[r] = __ldg(bits + ta + (uint64_t)(6 + r) * pitch); b1[r] = __ldg(bits + tb + (uint64_t)(6 + r) * pitch);
    }
    for (uint32_t j = 0; j < D; j++) {
      uint32_t a2[6], b2[6];
      const uint32_t jn = (j + 2 < D) ? j + 2 : j;
#pragma unroll
      for (int r = 0; r < 6; r++) {
        a2[r] = __ldg(bits + ta + ((uint64_t)jn * 6 + r) * pitch);
        b2[r] = __ldg(bits + tb + ((uint64_t)jn * 6 + r) * pitch);
      }
      walk64x2<V>(a0, b0, xa, ya, xb, yb, four);
      out[(uint64_t)j * W + ta] = ((uint64_t)ya << 32) | xa;
      out[(uint64_t)j * W + tb] = ((uint64_t)yb << 32) | xb;
#pragma unroll
      for (int r = 0; r < 6; r++) { a0[r] = a1[r]; a1[r] = a2[r]; b0[r] = b1[r]; b1[r] = b2[r]; }
    }
    xs[ta] = xa; ys[ta] = ya; xs[tb] = xb; ys[tb] = yb;
  }
}
__global__ void kinit(uint32_t* p, uint64_t n) {
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t z = i * 0x9E3779B97F4A7C15ull + 12345;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    p[i] = (uint32_t)z;
  }
}
template <int V>
float run2(const uint32_t* bits, uint64_t pitch, uint32_t W, uint32_t D, uint32_t* xs, uint32_t* ys, uint64_t* out,
           int warps_per_sm, int reps) {
  uint32_t units = W / 32;
  uint32_t max_warps = 148u * warps_per_sm;
  uint32_t k = (units / 2 + max_warps - 1) / max_warps;
  uint32_t warps = (units / 2 + k - 1) / k;
  uint32_t blocks = (warps + 1) / 2;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  kinit<<<1184, 256>>>(xs, W); kinit<<<1184, 256>>>(ys, W);
  cudaEventRecord(a);
  for (int r = 0; r < reps; r++) {
    kinit<<<1184, 256>>>(xs, W); kinit<<<1184, 256>>>(ys, W);
    kfill2<V><<<blocks, 64>>>(bits, pitch, W, D, xs, ys, out, units, 4u);
  }
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms / reps;
}

template <int NK>
__device__ __forceinline__ void word10x1U(uint32_t Qa, uint32_t &xa, uint32_t &ya) {
  uint32_t Ca, Fa;
  prep12(Qa, Ca, Fa);
  const uint32_t Ga = Fa >> 6;
  two13<0, 3, SH(0), SH(1)>(Fa, Ca, xa, ya);
  if (NK == 4) { two13<0, 3, SH(2), SH(3)>(Ga, Ca, xa, ya); return; }
  one13<0, SH(2)>(Ga, Ca, xa, ya);
  two13<9, 12, SH(3), SH(4)>(Fa, Ca, xa, ya);
  one13<9, SH(5)>(Ga, Ca, xa, ya);
  two13<18, 21, SH(6), SH(7)>(Fa, Ca, xa, ya);
  two13<24, 27, SH(8), SH(9)>(Fa, Ca, xa, ya);
}
template <int V, int NK>
__device__ __forceinline__ void word10x1V6(uint32_t Q, uint32_t &x, uint32_t &y) {
  const uint32_t f1 = Q >> 1, f2 = Q >> 2;
  const uint32_t MY = ~f2 & (f1 | Q), MX = f2 & ~(f1 & Q), C = Q - (MY & 0x09249249u);
#define S1(k) if (NK > k) step<6, k>(MY, MX, C, x, y, 4u);
  S1(0) S1(1) S1(2) S1(3) S1(4) S1(5) S1(6) S1(7) S1(8) S1(9)
#undef S1
}
template <int V>
__device__ __forceinline__ void walk64x1(const uint32_t a[6], uint32_t &x, uint32_t &y) {
#define W1(Q, NK) if (V == 13) word10x1U<NK>(Q, x, y); else word10x1V6<V, NK>(Q, x, y);
  W1(a[0], 10) W1(__funnelshift_r(a[0], a[1], 30), 10) W1(__funnelshift_r(a[1], a[2], 28), 10)
  W1(__funnelshift_r(a[2], a[3], 26), 10) W1(__funnelshift_r(a[3], a[4], 24), 10)
  W1(__funnelshift_r(a[4], a[5], 22), 10) W1(a[5] >> 20, 4)
#undef W1
}
template <int V>
__global__ void __launch_bounds__(64) kfill1(const uint32_t* __restrict__ bits, uint64_t pitch, uint32_t W, uint32_t D,
                                             uint32_t* xs, uint32_t* ys, uint64_t* out, uint32_t units, uint32_t four) {
  const uint32_t lane = threadIdx.x & 31u, warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t u = warp; u < units; u += nwarps) {
    const uint32_t t = u * 32u + lane;
    uint32_t x = xs[t], y = ys[t];
    uint32_t w0[6], w1[6];
#pragma unroll
    for (int r = 0; r < 6; r++) { w0[r] = __ldg(bits + t + (uint64_t)r * pitch); w1[r] = __ldg(bits + t + (uint64_t)(6 + r) * pitch); }
    for (uint32_t j = 0; j < D; j++) {
      uint32_t w2[6];
      const uint32_t jn = (j + 2 < D) ? j + 2 : j;
#pragma unroll
      for (int r = 0; r < 6; r++) w2[r] = __ldg(bits + t + ((uint64_t)jn * 6 + r) * pitch);
      walk64x1<V>(w0, x, y);
      out[(uint64_t)j * W + t] = ((uint64_t)y << 32) | x;
#pragma unroll
      for (int r = 0; r < 6; r++) { w0[r] = w1[r]; w1[r] = w2[r]; }
    }
    xs[t] = x; ys[t] = y;
  }
}
template <int V>
float run1(const uint32_t* bits, uint64_t pitch, uint32_t W, uint32_t D, uint32_t* xs, uint32_t* ys, uint64_t* out,
           int warps_per_sm, int reps) {
  uint32_t units = W / 32;
  uint32_t max_warps = 148u * warps_per_sm;
  uint32_t k = (units + max_warps - 1) / max_warps;
  uint32_t warps = (units + k - 1) / k;
  uint32_t blocks = (warps + 1) / 2;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  for (int r = 0; r < reps; r++) {
    kinit<<<1184, 256>>>(xs, W); kinit<<<1184, 256>>>(ys, W);
    kfill1<V><<<blocks, 64>>>(bits, pitch, W, D, xs, ys, out, units, 4u);
  }
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms / reps;
}

// NW walkers per thread (t = u*32*NW + k*32 + lane), R2P step; groups interleaved across walkers.
template <int NW, int NK>
__device__ __forceinline__ void wordN(const uint32_t (&Q)[NW], uint32_t (&x)[NW], uint32_t (&y)[NW]) {
  uint32_t C[NW], F[NW], G[NW];
#pragma unroll
  for (int k = 0; k < NW; k++) { prep12(Q[k], C[k], F[k]); G[k] = F[k] >> 6; }
#define AW2(B0, B1, K0, K1, S) _Pragma("unroll") for (int k = 0; k < NW; k++) two13<B0, B1, SH(K0), SH(K1)>(S[k], C[k], x[k], y[k]);
#define AW1(B0, K0, S) _Pragma("unroll") for (int k = 0; k < NW; k++) one13<B0, SH(K0)>(S[k], C[k], x[k], y[k]);
  AW2(0, 3, 0, 1, F)
  if (NK == 4) { AW2(0, 3, 2, 3, G) return; }
  AW1(0, 2, G) AW2(9, 12, 3, 4, F) AW1(9, 5, G) AW2(18, 21, 6, 7, F) AW2(24, 27, 8, 9, F)
#undef AW2
#undef AW1
}
template <int NW>
__device__ __forceinline__ void walkN(const uint32_t (&w)[NW][6], uint32_t (&x)[NW], uint32_t (&y)[NW]) {
  uint32_t Q[NW];
#pragma unroll
  for (int k = 0; k < NW; k++) Q[k] = w[k][0];
  wordN<NW, 10>(Q, x, y);
#pragma unroll
  for (int i = 1; i < 6; i++) {
#pragma unroll
    for (int k = 0; k < NW; k++) Q[k] = __funnelshift_r(w[k][i - 1], w[k][i], 32 - 2 * i);
    wordN<NW, 10>(Q, x, y);
  }
#pragma unroll
  for (int k = 0; k < NW; k++) Q[k] = w[k][5] >> 20;
  wordN<NW, 4>(Q, x, y);
}
template <int NW, int MINB>
__global__ void __launch_bounds__(64, MINB) kfillN(const uint32_t* __restrict__ bits, uint64_t pitch, uint32_t W, uint32_t D,
                                             uint32_t* xs, uint32_t* ys, uint64_t* out, uint32_t units, uint32_t four) {
  const uint32_t lane = threadIdx.x & 31u, warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t u = warp; u < units / NW; u += nwarps) {
    uint32_t x[NW], y[NW], w0[NW][6], w1[NW][6];
#pragma unroll
    for (int k = 0; k < NW; k++) {
      const uint32_t t = u * 32u * NW + k * 32u + lane;
      x[k] = xs[t]; y[k] = ys[t];
#pragma unroll
      for (int r = 0; r < 6; r++) { w0[k][r] = __ldg(bits + t + (uint64_t)r * pitch); w1[k][r] = __ldg(bits + t + (uint64_t)(6 + r) * pitch); }
    }
    for (uint32_t j = 0; j < D; j++) {
      uint32_t w2[NW][6];
      const uint32_t jn = (j + 2 < D) ? j + 2 : j;
#pragma unroll
      for (int k = 0; k < NW; k++) {
        const uint32_t t = u * 32u * NW + k * 32u + lane;
#pragma unroll
        for (int r = 0; r < 6; r++) w2[k][r] = __ldg(bits + t + ((uint64_t)jn * 6 + r) * pitch);
      }
      walkN<NW>(w0, x, y);
#pragma unroll
      for (int k = 0; k < NW; k++) {
        const uint32_t t = u * 32u * NW + k * 32u + lane;
        out[(uint64_t)j * W + t] = ((uint64_t)y[k] << 32) | x[k];
#pragma unroll
        for (int r = 0; r < 6; r++) { w0[k][r] = w1[k][r]; w1[k][r] = w2[k][r]; }
      }
    }
#pragma unroll
    for (int k = 0; k < NW; k++) { const uint32_t t = u * 32u * NW + k * 32u + lane; xs[t] = x[k]; ys[t] = y[k]; }
  }
}
template <int NW, int MINB>
float runN(const uint32_t* bits, uint64_t pitch, uint32_t W, uint32_t D, uint32_t* xs, uint32_t* ys, uint64_t* out,
           int reps) {
  uint32_t units = W / 32;
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfillN<NW, MINB>, 64, 0);
  uint32_t max_warps = 148u * per_sm * 2;
  uint32_t k = (units / NW + max_warps - 1) / max_warps;
  uint32_t warps = (units / NW + k - 1) / k;
  uint32_t blocks = (warps + 1) / 2;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  for (int r = 0; r < reps; r++) {
    kinit<<<1184, 256>>>(xs, W); kinit<<<1184, 256>>>(ys, W);
    kfillN<NW, MINB><<<blocks, 64>>>(bits, pitch, W, D, xs, ys, out, units, 4u);
  }
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms / reps;
}
int main(int argc, char** argv) {
  const uint32_t W = 1u << 20, D = 128;
  const int reps = argc > 1 ? atoi(argv[1]) : 5;
  const uint64_t pitch = W;
  uint32_t *bits, *xs, *ys; uint64_t* out;
  cudaMalloc(&bits, (size_t)D * 6 * pitch * 4);
  cudaMalloc(&xs, W * 4); cudaMalloc(&ys, W * 4);
  cudaMalloc(&out, (size_t)D * W * 8);
  kinit<<<4096, 256>>>(bits, (uint64_t)D * 6 * pitch);
  std::vector<uint64_t> ref(W), got(W);
  double labels = (double)W * D;
  for (int wps : {16, 24, 32}) {
    float t6 = run2<6>(bits, pitch, W, D, xs, ys, out, wps, reps);
    cudaMemcpy(ref.data(), out + (size_t)(D - 1) * W, W * 8, cudaMemcpyDeviceToHost);
    printf("warps/SM %d: V6 %.3f ms (%.1f G/s)", wps, t6, labels / t6 / 1e6);
#define VAR(v) { float t = run2<v>(bits, pitch, W, D, xs, ys, out, wps, reps); \
      cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, W * 8, cudaMemcpyDeviceToHost); \
      printf("  V%d %.3f (%.1f) %s", v, t, labels / t / 1e6, got == ref ? "ok" : "MISMATCH"); }
    VAR(13) VAR(14)
    printf("\n");
  }
  for (int wps : {32, 48, 64}) {
    float t6 = run1<6>(bits, pitch, W, D, xs, ys, out, wps, reps);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, W * 8, cudaMemcpyDeviceToHost);
    bool ok6 = got == ref;
    float t13 = run1<13>(bits, pitch, W, D, xs, ys, out, wps, reps);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, W * 8, cudaMemcpyDeviceToHost);
    printf("x1 warps/SM %d: V6 %.3f (%.1f) %s  V13 %.3f (%.1f) %s\n", wps, t6, labels / t6 / 1e6, ok6 ? "ok" : "MISMATCH",
           t13, labels / t13 / 1e6, got == ref ? "ok" : "MISMATCH");
  }
#define RN(NW, MB) { float t = runN<NW, MB>(bits, pitch, W, D, xs, ys, out, reps); \
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, W * 8, cudaMemcpyDeviceToHost); \
    int per_sm = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfillN<NW, MB>, 64, 0); \
    printf("N=%d minb=%d (%d blk/SM): %.3f ms (%.1f G/s) %s\n", NW, MB, per_sm, t, labels / t / 1e6, got == ref ? "ok" : "MISMATCH"); }
  RN(1, 1) RN(2, 1) RN(2, 16) RN(2, 24) RN(3, 1) RN(3, 12) RN(4, 1) RN(4, 8)
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
