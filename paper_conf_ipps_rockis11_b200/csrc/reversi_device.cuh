// reversi_device.cuh — device game core for the playout hot loop (sm_100a).
//
// Bitboard 8x8 Reversi: square s = 8*row + col, bit s of a uint64 (DESIGN.md
// §3 R7). Everything here is plain integer/bit work on the ALU and FMA pipes:
// shift-mask move generation, a branch-free popc binary search for the random
// pick, shift-mask flips and a counter-based Philox4x32-10. See DESIGN.md §6
// for the per-ply instruction budget these functions set.
//
// PAPER.md L149-L151 (§II): "A simulation is defined as a series of random
// moves which are performed until the end of a game is reached (until neither
// of the players can move)."
#pragma once
#include <cstdint>

namespace mcts_dev {

typedef unsigned long long u64;
typedef uint32_t u32;

// Propagator mask for directions with a column component: an opponent disc on
// file a or h can never be bracketed along a horizontal or diagonal line.
constexpr u64 kInner = 0x7E7E7E7E7E7E7E7EULL;

template <int S>
__device__ __forceinline__ u64 sh(u64 x) {
  if constexpr (S > 0) return x << S;
  else return x >> (-S);
}

// Moves of P against O along direction S: a run of >= 1 propagator discs M
// attached to P, continued by one more step (the landing square). 6 fill steps
// cover the longest possible run (6 discs between two squares of a line).
template <int S>
__device__ __forceinline__ u64 dir_moves(u64 P, u64 M) {
  u64 t = M & sh<S>(P);
  t |= M & sh<S>(t);
  t |= M & sh<S>(t);
  t |= M & sh<S>(t);
  t |= M & sh<S>(t);
  t |= M & sh<S>(t);
  return sh<S>(t);
}

// Legal-move mask of the side owning P (opponent O).
__device__ __forceinline__ u64 legal_moves(u64 P, u64 O) {
  const u64 M = O & kInner;
  u64 m = dir_moves<1>(P, M) | dir_moves<-1>(P, M);
  m |= dir_moves<8>(P, O) | dir_moves<-8>(P, O);
  m |= dir_moves<7>(P, M) | dir_moves<-7>(P, M);
  m |= dir_moves<9>(P, M) | dir_moves<-9>(P, M);
  return m & ~(P | O);
}

// Discs flipped along direction S when P plays the square x (a single bit):
// the contiguous propagator run starting next to x, kept only if the square
// after it holds a P disc.
template <int S>
__device__ __forceinline__ u64 dir_flips(u64 x, u64 P, u64 M) {
  u64 t = M & sh<S>(x);
  t |= M & sh<S>(t);
  t |= M & sh<S>(t);
  t |= M & sh<S>(t);
  t |= M & sh<S>(t);
  t |= M & sh<S>(t);
  return (sh<S>(t) & P) ? t : 0ULL;
}

__device__ __forceinline__ u64 flips(int sq, u64 P, u64 O) {
  const u64 x = 1ULL << sq;
  const u64 M = O & kInner;
  u64 f = dir_flips<1>(x, P, M) | dir_flips<-1>(x, P, M);
  f |= dir_flips<8>(x, P, O) | dir_flips<-8>(x, P, O);
  f |= dir_flips<7>(x, P, M) | dir_flips<-7>(x, P, M);
  f |= dir_flips<9>(x, P, M) | dir_flips<-9>(x, P, M);
  return f;
}

// ---------------------------------------------------------------------------
// Hot-loop variants (same results as legal_moves / flips, fewer ALU-pipe slots).
//
// The playout loop is integer-issue bound and, compiled naively, saturates the
// ALU pipe (LOP3/SHF/IADD3/SEL, 16 lanes/SMSP/clk) while the FMA pipe (IMAD,
// also 16 lanes/SMSP/clk) idles. Shifting by multiplying with a power of two
// runs on the FMA pipe; the multipliers live in constant memory so ptxas cannot
// fold them back into SHF. Each shift helper picks its pipe mix by template
// argument:
//   shl<S, kAlu>: IMAD.SHL + SHF        shl<S, kFma>: IMAD.WIDE + IMAD
//   shr<S, kAlu>: 2 x SHF               shr<S, kMix>: SHF + IMAD.HI
//   shr<S, kFma>: IMAD.HI + IMAD + IMAD.HI
__constant__ u32 c_pow2[33] = {
    1u, 2u, 4u, 8u, 16u, 32u, 64u, 128u, 256u, 512u, 1024u, 2048u, 4096u, 8192u, 16384u, 32768u,
    1u << 16, 1u << 17, 1u << 18, 1u << 19, 1u << 20, 1u << 21, 1u << 22, 1u << 23, 1u << 24,
    1u << 25, 1u << 26, 1u << 27, 1u << 28, 1u << 29, 1u << 30, 1u << 31, 0u};

enum { kAlu = 0, kFma = 1, kMix = 2 };

// Pipe-mix configuration of the hot loop (tuned on B200).
#ifndef MCTS_MG_LEFT
#define MCTS_MG_LEFT kAlu
#endif
#ifndef MCTS_MG_RIGHT
#define MCTS_MG_RIGHT kAlu
#endif
#ifndef MCTS_MG_EAST_CARRY
#define MCTS_MG_EAST_CARRY 1
#endif
#ifndef MCTS_EAST_PLAIN
#define MCTS_EAST_PLAIN 0
#endif
#ifndef MCTS_PICK_F
#define MCTS_PICK_F 0
#endif
#ifndef MCTS_UPD_F
#define MCTS_UPD_F 1
#endif
#ifndef MCTS_FLIP_ADD_F
#define MCTS_FLIP_ADD_F 0
#endif
#ifndef MCTS_MG_REVERSED
#define MCTS_MG_REVERSED 1
#endif
// per-step shift pipe of up_moves (kAlu: IMAD.SHL + funnel SHF; kFma: IMAD.WIDE + IMAD)
#ifndef MCTS_UP_M2
#define MCTS_UP_M2 kAlu
#endif
#ifndef MCTS_UP_S1
#define MCTS_UP_S1 kAlu
#endif
#ifndef MCTS_UP_S2
#define MCTS_UP_S2 kAlu
#endif
#ifndef MCTS_UP_D1
#define MCTS_UP_D1 kAlu
#endif
#ifndef MCTS_UP_D2
#define MCTS_UP_D2 kAlu
#endif
#ifndef MCTS_UP_FIN
#define MCTS_UP_FIN kAlu
#endif
#ifndef MCTS_PICK_LUT
#define MCTS_PICK_LUT 1
#endif
#ifndef MCTS_RNG_SELECT
#define MCTS_RNG_SELECT 0
#endif

__device__ __forceinline__ u64 join32(u32 lo, u32 hi) { return ((u64)hi << 32) | lo; }

template <int S, int MODE>
__device__ __forceinline__ u64 shl(u64 x) {
  static_assert(S > 0 && S < 32, "shift");
  if constexpr (MODE == kAlu) {
    return x << S;
  } else {
    const u32 lo = (u32)x, hi = (u32)(x >> 32), m = c_pow2[S];
    return join32(lo * m, hi * m + __umulhi(lo, m));
  }
}

template <int S, int MODE>
__device__ __forceinline__ u64 shr(u64 x) {
  static_assert(S > 0 && S < 32, "shift");
  const u32 lo = (u32)x, hi = (u32)(x >> 32);
  if constexpr (MODE == kAlu) {
    return x >> S;
  } else if constexpr (MODE == kMix) {
    return join32(__funnelshift_r(lo, hi, S), __umulhi(hi, c_pow2[32 - S]));
  } else {
    const u32 m = c_pow2[32 - S];
    return join32(hi * m + __umulhi(lo, m), __umulhi(hi, m));
  }
}

// Move generation with a shared doubled propagator: after two single steps the
// run from P covers 2 squares, after two double steps (M2 = M & M<<S) it covers
// 6, the longest possible run. M2 for -S is M2 >> S, so an axis costs one M2.
template <int S, int LM, int RM>
__device__ __forceinline__ u64 axis_moves(u64 P, u64 M) {
  const u64 M2 = M & shl<S, LM>(M);
  u64 t = M & shl<S, LM>(P);
  t |= M & shl<S, LM>(t);
  t |= M2 & shl<2 * S, LM>(t);
  t |= M2 & shl<2 * S, LM>(t);
  const u64 M2r = shr<S, RM>(M2);
  u64 u = M & shr<S, RM>(P);
  u |= M & shr<S, RM>(u);
  u |= M2r & shr<2 * S, RM>(u);
  u |= M2r & shr<2 * S, RM>(u);
  return shl<S, LM>(t) | shr<S, RM>(u);
}

__device__ __forceinline__ u64 legal_moves_fast(u64 P, u64 O) {
  const u64 M = O & kInner;
  u64 m = axis_moves<1, kFma, kMix>(P, M);
  m |= axis_moves<8, kFma, kFma>(P, O);
  m |= axis_moves<7, kFma, kMix>(P, M);
  m |= axis_moves<9, kFma, kFma>(P, M);
  return m & ~(P | O);
}

// Upward ray masks (squares strictly beyond sq in direction +1, +8, +7, +9 up
// to the board edge) and the ray's first square, in a per-CTA shared table:
// rays[d*64 + sq] = mask, rays[256 + d*64 + sq] = first square (0 at an edge).
__device__ __forceinline__ u64 ray_mask(int dir_index, int sq) {
  const int dr = dir_index == 0 ? 0 : 1;
  const int dc = dir_index == 1 ? 0 : (dir_index == 2 ? -1 : 1);
  int r = sq >> 3, c = sq & 7;
  u64 m = 0;
  for (;;) {
    r += dr;
    c += dc;
    if (r < 0 || r > 7 || c < 0 || c > 7) break;
    m |= 1ULL << (8 * r + c);
  }
  return m;
}

// Shared per-CTA table: [0,256) ray masks, [256,512) first ray squares,
// [512,768) a byte-select LUT: byte (k*256 + b) = index of the k-th set bit of b.
constexpr int kRayTable = 768;

// Flips along an upward ray by carry propagation: adding the ray's first square
// to (O | ~m) carries through the contiguous opponent run (and through the
// non-ray bits, all ones) and lands on the first non-opponent ray square.
// run = ray squares that carried (~s & O & m); kept iff the landing square is P.
// The 64-bit add runs on the FMA pipe (IMAD.WIDE by one, then IMAD on the high
// word: first is a single bit, so at most one of its halves is non-zero).
__device__ __forceinline__ void up_flips(u64& f, u64 first, u64 P, u64 O, u64 m, u32 one) {
  const u64 xo = O | ~m;
#if MCTS_FLIP_ADD_F
  const u64 s0 = (u64)((u32)first) * one + xo;
  const u64 s = join32((u32)s0, (u32)(first >> 32) * one + (u32)(s0 >> 32));
#else
  const u64 s = xo + first;
#endif
  if (s & m & P) f |= ~s & O & m;
}

// All 8 directions: the 4 upward ones directly, the 4 downward ones as upward
// directions of the 180-degree-rotated (bit-reversed) board, where square sq
// becomes 63 - sq and the same table applies.
__device__ __forceinline__ u64 flips_fast(int sq, u64 P, u64 O, const u64* __restrict__ rays) {
  const u32 one = c_pow2[0];
  u64 f = 0;
  up_flips(f, rays[256 + sq], P, O, rays[sq], one);
  up_flips(f, rays[320 + sq], P, O, rays[64 + sq], one);
  up_flips(f, rays[384 + sq], P, O, rays[128 + sq], one);
  up_flips(f, rays[448 + sq], P, O, rays[192 + sq], one);
  const int rs = 63 - sq;
  const u64 rP = __brevll(P), rO = __brevll(O);
  u64 g = 0;
  up_flips(g, rays[256 + rs], rP, rO, rays[rs], one);
  up_flips(g, rays[320 + rs], rP, rO, rays[64 + rs], one);
  up_flips(g, rays[384 + rs], rP, rO, rays[128 + rs], one);
  up_flips(g, rays[448 + rs], rP, rO, rays[192 + rs], one);
  return f | __brevll(g);
}

// ---- FMA-pipe integer helpers (the multiplier 1 comes from constant memory
// so ptxas keeps IMAD rather than an ALU-pipe IADD3) ----------------------------
__device__ __forceinline__ u32 add_f(u32 a, u32 b) { return a * c_pow2[0] + b; }   // a + b
__device__ __forceinline__ u32 sub_f(u32 a, u32 b) { return b * (0u - c_pow2[0]) + a; }  // a - b
// Disjoint 64-bit add / subset subtract as two independent 32-bit IMADs:
// a | b when a & b == 0, and a & ~b when b is a subset of a.
__device__ __forceinline__ u64 or_disjoint_f(u64 a, u64 b) {
  return join32(add_f((u32)a, (u32)b), add_f((u32)(a >> 32), (u32)(b >> 32)));
}
__device__ __forceinline__ u64 andnot_subset_f(u64 a, u64 b) {
  return join32(sub_f((u32)a, (u32)b), sub_f((u32)(a >> 32), (u32)(b >> 32)));
}

// Horizontal (+1) moves by carry propagation, per 32-bit half (a row never
// spans halves and no carry leaves a row: the landing square of a run ending
// on column 6 is column 7, and column 7 is never in M). t = P<<1 per half;
// s = M + t carries each adjacent opponent run to its landing square; s & ~t
// keeps landings (and non-carried O / P squares, removed by the final empty
// mask of the caller).
__device__ __forceinline__ u64 east_moves_f(u64 P, u64 M) {
#if MCTS_EAST_PLAIN
  const u32 tl = (u32)P << 1, th = (u32)(P >> 32) << 1;
  const u32 sl = (u32)M + tl, sh_ = (u32)(M >> 32) + th;
#else
  const u32 two = c_pow2[1];
  const u32 tl = (u32)P * two, th = (u32)(P >> 32) * two;
  const u32 sl = add_f((u32)M, tl), sh_ = add_f((u32)(M >> 32), th);
#endif
  return join32(sl & ~tl, sh_ & ~th);
}

// One upward direction (+S, S in {7, 8, 9}) of the doubled-propagator fill,
// left shifts only (lo: IMAD.SHL on the FMA pipe, hi: one funnel SHF).
template <int S>
__device__ __forceinline__ u64 up_moves(u64 P, u64 M) {
  const u64 M2 = M & shl<S, MCTS_UP_M2>(M);
  u64 t = M & shl<S, MCTS_UP_S1>(P);
  t |= M & shl<S, MCTS_UP_S2>(t);
  t |= M2 & shl<2 * S, MCTS_UP_D1>(t);
  t |= M2 & shl<2 * S, MCTS_UP_D2>(t);
  return shl<S, MCTS_UP_FIN>(t);
}

// Legal moves. The four upward directions (+1 by carries, +7/+8/+9 by fills)
// run on the board; the four downward ones run as upward directions of the
// bit-reversed board rP/rO (square s -> 63 - s is the 180-degree rotation, so
// -1/-7/-8/-9 become +1/+7/+8/+9 and the file masks are unchanged). Only left
// shifts remain, which split evenly between the ALU and FMA pipes; the caller
// reuses rP/rO for the flips.
__device__ __forceinline__ u64 legal_moves_hot(u64 P, u64 O, u64 rP, u64 rO) {
#if MCTS_MG_REVERSED
  const u64 M = O & kInner, rM = rO & kInner;
  u64 m = east_moves_f(P, M);
  m |= up_moves<8>(P, O);
  m |= up_moves<7>(P, M);
  m |= up_moves<9>(P, M);
  u64 r = east_moves_f(rP, rM);
  r |= up_moves<8>(rP, rO);
  r |= up_moves<7>(rP, rM);
  r |= up_moves<9>(rP, rM);
  return (m | __brevll(r)) & ~(P | O);
#else
  const u64 M = O & kInner;
#if MCTS_MG_EAST_CARRY
  u64 m = east_moves_f(P, M);
  m |= __brevll(east_moves_f(rP, rO & kInner));
#else
  u64 m = axis_moves<1, MCTS_MG_LEFT, MCTS_MG_RIGHT>(P, M);
#endif
  m |= axis_moves<8, MCTS_MG_LEFT, MCTS_MG_RIGHT>(P, O);
  m |= axis_moves<7, MCTS_MG_LEFT, MCTS_MG_RIGHT>(P, M);
  m |= axis_moves<9, MCTS_MG_LEFT, MCTS_MG_RIGHT>(P, M);
  return m & ~(P | O);
#endif
}

// flips_fast with the bit-reversed board supplied by the caller.
__device__ __forceinline__ u64 flips_hot(int sq, u64 P, u64 O, u64 rP, u64 rO,
                                         const u64* __restrict__ rays) {
  const u32 one = c_pow2[0];
  u64 f = 0;
  up_flips(f, rays[256 + sq], P, O, rays[sq], one);
  up_flips(f, rays[320 + sq], P, O, rays[64 + sq], one);
  up_flips(f, rays[384 + sq], P, O, rays[128 + sq], one);
  up_flips(f, rays[448 + sq], P, O, rays[192 + sq], one);
  const int rs = 63 - sq;
  u64 g = 0;
  up_flips(g, rays[256 + rs], rP, rO, rays[rs], one);
  up_flips(g, rays[320 + rs], rP, rO, rays[64 + rs], one);
  up_flips(g, rays[384 + rs], rP, rO, rays[128 + rs], one);
  up_flips(g, rays[448 + rs], rP, rO, rays[192 + rs], one);
  return f | __brevll(g);
}

// k-th set bit with the selects done arithmetically on the FMA pipe:
// per level s = (k < c) in {0,1} from the sign of k - c, then
// x = hi + s*(lo - hi), k = (k - c) + s*c, base += W*(1 - s).
__device__ __forceinline__ int kth_set_bit_f(u64 m, u32 k) {
  const u32 one = c_pow2[0];
  u32 x = (u32)m;
  const u32 hi = (u32)(m >> 32);
  u32 c = __popc(x);
  u32 d = sub_f(k, c);
  u32 sgn = __umulhi(d, c_pow2[1]);  // (k - c) >> 31: 1 iff k < c
  x = sgn * (x - hi) + hi;
  k = sgn * c + d;
  u32 base = sgn * (0u - 32u * one) + 32u;
#pragma unroll
  for (int wdt = 16; wdt >= 2; wdt >>= 1) {
    const u32 lowm = x & ((1u << wdt) - 1u);
    c = __popc(lowm);
    d = sub_f(k, c);
    sgn = __umulhi(d, c_pow2[1]);
    // upper part: x >> wdt on the FMA pipe
    const u32 up = __umulhi(x, c_pow2[32 - wdt]);
    x = sgn * (lowm - up) + up;
    k = sgn * c + d;
    base = sgn * (0u - (u32)wdt * one) + (base + (u32)wdt);
  }
  // last level (width 1): bit 0 of x is set iff c = 1
  c = x & 1u;
  d = sub_f(k, c);
  sgn = __umulhi(d, c_pow2[1]);
  base = sgn * (0u - one) + (base + 1u);
  return (int)base;
}

// Index (0..63) of the k-th set bit (k = 0: lowest) of m; k < popc(m).
// Branch-free binary search on population counts.
__device__ __forceinline__ int kth_set_bit(u64 m, u32 k) {
  u32 lo = (u32)m, hi = (u32)(m >> 32);
  u32 c = __popc(lo);
  bool up = k >= c;
  u32 x = up ? hi : lo;
  k -= up ? c : 0u;
  int base = up ? 32 : 0;
  c = __popc(x & 0xFFFFu); up = k >= c; x = up ? (x >> 16) : x; k -= up ? c : 0u; base += up ? 16 : 0;
  c = __popc(x & 0xFFu);   up = k >= c; x = up ? (x >> 8) : x;  k -= up ? c : 0u; base += up ? 8 : 0;
  c = __popc(x & 0xFu);    up = k >= c; x = up ? (x >> 4) : x;  k -= up ? c : 0u; base += up ? 4 : 0;
  c = __popc(x & 0x3u);    up = k >= c; x = up ? (x >> 2) : x;  k -= up ? c : 0u; base += up ? 2 : 0;
  c = x & 1u;              up = k >= c;                                           base += up ? 1 : 0;
  return base;
}

// k-th set bit: three popc levels down to a byte, then the byte-select LUT.
__device__ __forceinline__ int kth_set_bit_lut(u64 m, u32 k, const unsigned char* __restrict__ lut) {
  u32 lo = (u32)m, hi = (u32)(m >> 32);
  u32 c = __popc(lo);
  bool up = k >= c;
  u32 x = up ? hi : lo;
  k -= up ? c : 0u;
  int base = up ? 32 : 0;
  c = __popc(x & 0xFFFFu); up = k >= c; x = up ? (x >> 16) : x; k -= up ? c : 0u; base += up ? 16 : 0;
  c = __popc(x & 0xFFu);   up = k >= c; x = up ? (x >> 8) : x;  k -= up ? c : 0u; base += up ? 8 : 0;
  return base + lut[(k << 8) | (x & 0xFFu)];
}

// Uniform pick (R4): k = floor(r * c / 2^32), then the k-th legal
// square in ascending order.
__device__ __forceinline__ int pick_square(u64 moves, u32 r) {
  u32 c = (u32)__popcll(moves);
  return kth_set_bit(moves, __umulhi(r, c));
}

// Philox4x32-10 (Salmon et al. SC'11; cuRAND/Random123 round and constants).
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
#pragma unroll
  for (int i = 0; i < 10; ++i) {
    const u32 hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    const u32 hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
    k.x += 0x9E3779B9u;
    k.y += 0xBB67AE85u;
  }
  return c;
}

// Stream of RNG words for one playout (R5): word w is output[w % 4]
// of Philox(counter = (c0, c1, c2, w / 4), key = seed).
struct PlayoutRng {
  uint2 key;
  u32 c0, c1, c2;
  u32 w;
  uint4 buf;  // the unread words of the current Philox block, in order
  __device__ __forceinline__ u32 next() {
#if MCTS_RNG_SELECT
    const u32 lane = w & 3u;
    if (lane == 0u) buf = philox4x32_10(make_uint4(c0, c1, c2, w >> 2), key);
    ++w;
    u32 r = buf.x;
    r = lane == 1u ? buf.y : r;
    r = lane == 2u ? buf.z : r;
    r = lane == 3u ? buf.w : r;
    return r;
#else
    if ((w & 3u) == 0u) buf = philox4x32_10(make_uint4(c0, c1, c2, w >> 2), key);
    ++w;
    const u32 r = buf.x;
    buf.x = buf.y;
    buf.y = buf.z;
    buf.z = buf.w;
    return r;
#endif
  }
};

// One decision for the side owning P: returns false if P has no move (a pass;
// nothing changes), else plays the random move and returns true.
__device__ __forceinline__ bool ply(u64& P, u64& O, PlayoutRng& rng, const u64* __restrict__ rays) {
  const u64 rP = __brevll(P), rO = __brevll(O);
  const u64 moves = legal_moves_hot(P, O, rP, rO);
  if (moves == 0ULL) return false;
  const u32 r = rng.next();
#if MCTS_PICK_F
  const int sq = kth_set_bit_f(moves, __umulhi(r, (u32)__popcll(moves)));
#elif MCTS_PICK_LUT
  const int sq = kth_set_bit_lut(moves, __umulhi(r, (u32)__popcll(moves)),
                                 reinterpret_cast<const unsigned char*>(rays + 512));
#else
  const int sq = kth_set_bit(moves, __umulhi(r, (u32)__popcll(moves)));
#endif
  const u64 f = flips_hot(sq, P, O, rP, rO, rays);
#if MCTS_UPD_F
  P = or_disjoint_f(P, or_disjoint_f(f, 1ULL << sq));
  O = andnot_subset_f(O, f);
#else
  P |= f | (1ULL << sq);
  O &= ~f;
#endif
  return true;
}

// One random playout from (me to move, op). Returns +1 / 0 / -1 for the side
// to move at the start (R3), adds the non-pass plies to *plies.
// A pass consumes no RNG word; two consecutive passes end the game. The loop is
// unrolled by two so the sides keep their registers (no swaps).
__device__ __forceinline__ int playout(u64 me, u64 op, uint2 key, u32 c0, u32 c1, u32 c2,
                                       const u64* __restrict__ rays, u32* plies) {
  PlayoutRng rng;
  rng.key = key; rng.c0 = c0; rng.c1 = c1; rng.c2 = c2; rng.w = 0;
  rng.buf = make_uint4(0, 0, 0, 0);
  bool passed = false;
  u32 n = 0;
  for (;;) {
    if (ply(me, op, rng, rays)) { passed = false; ++n; }
    else if (passed) break;  // neither player can move
    else passed = true;
    if (ply(op, me, rng, rays)) { passed = false; ++n; }
    else if (passed) break;
    else passed = true;
  }
  *plies += n;
  const int a = __popcll(me), b = __popcll(op);
  return (a > b) - (a < b);
}

// Fill the per-CTA shared ray table (4 x 64 u64) used by flips_fast; every
// thread of the block must call it, followed by __syncthreads().
__device__ __forceinline__ void fill_rays(u64* rays) {
  for (int i = threadIdx.x; i < 256; i += blockDim.x) {
    const u64 m = ray_mask(i >> 6, i & 63);
    rays[i] = m;
    rays[256 + i] = m & (0ULL - m);  // lowest ray square (0 if the ray is empty)
    u64 packed = 0;                  // LUT bytes 8i .. 8i+7
    for (int j = 0; j < 8; ++j) {
      const int e = 8 * i + j, k = e >> 8, b = e & 255;
      int seen = 0, pos = 0;
      for (int q = 0; q < 8; ++q)
        if ((b >> q) & 1) { if (seen == k) { pos = q; break; } ++seen; }
      packed |= (u64)pos << (8 * j);
    }
    rays[512 + i] = packed;
  }
}

// Terminal test: neither side has a move.
__device__ __forceinline__ bool is_terminal(u64 P, u64 O, u64 legalP) {
  return legalP == 0ULL && legal_moves(O, P) == 0ULL;
}

}  // namespace mcts_dev
