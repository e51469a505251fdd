// reversi_device.cuh — device game core for the playout hot loop (sm_100a).
//
// Bitboard 8x8 Reversi: square s = 8*row + col, bit s of a uint64 (DESIGN.md
// §3 R7). PAPER.md L149-L151 (§II): "A simulation is defined as a series of
// random moves which are performed until the end of a game is reached (until
// neither of the players can move)."
//
// Two layers:
//   * plain reference-style functions (legal_moves, flips, kth_set_bit) used by
//     the tree code and the input generator, where speed does not matter;
//   * the hot ply loop (legal_moves_hot, flips_loop, kth_set_bit_lut, ply,
//     playout), shaped for the B200 integer pipes — see DESIGN.md §5-§6: the
//     loop is bound by the ALU pipe (LOP3/SHF/IADD3/SEL, 16 lanes/SMSP/clk), so
//     it is written to need as few ALU-pipe instructions as possible: downward
//     directions run as upward ones on the bit-reversed board (left shifts are
//     IMADs by 2^S on the FMA pipe), vertical/diagonal move fills run on 32-bit
//     words with one cross term, horizontal moves and all flips use carries,
//     and the flips of the frame whose move lies in the hi word are 32-bit.
#pragma once
#include <cstdint>

// Tuning knobs (defaults = the measured best on B200; tools/build_variants.py).
#ifndef MCTS_PICK_LUT
#define MCTS_PICK_LUT 1  // byte-select LUT for the last 3 levels of the k-th-bit search
#endif
#ifndef MCTS_UPD_F
#define MCTS_UPD_F 1     // board update as disjoint IMAD adds/subtracts
#endif
#ifndef MCTS_EAST_F
#define MCTS_EAST_F 1    // horizontal carry moves with IMAD shifts/adds
#endif
#ifndef MCTS_SPLIT
#define MCTS_SPLIT 1     // vertical/diagonal move fills on 32-bit halves (one cross term per direction)
#endif
#ifndef MCTS_FLIP_XY
#define MCTS_FLIP_XY 1   // flips with one frame's rays on 32-bit words (see flips_hot_xy)
#endif
#ifndef MCTS_BIT_LUT
#define MCTS_BIT_LUT 1   // 1 << sq from the shared table
#endif
#ifndef MCTS_PICK_SHL
#define MCTS_PICK_SHL 0  // k-th bit: popc of the low 16/8 bits as popc(x << 16/24) (IMAD) instead of a mask (LOP3)
#endif
#ifndef MCTS_MAPBACK3
#define MCTS_MAPBACK3 0  // flips back to board coordinates with 3 BREV and 2 SEL per word pair instead of 2 BREV + 4 SEL
#endif
#ifndef MCTS_RM_BREV
#define MCTS_RM_BREV 1   // reversed-board propagator mask as brev(O & inner) (XU) instead of rO & inner (ALU)
#endif
#ifndef MCTS_HXP
#define MCTS_HXP 1       // the flips' frame (square >= 32) taken from the pick's first popc level
#endif
#ifndef MCTS_NW
#define MCTS_NW 1        // the ply counter doubles as the RNG word index (one increment per ply)
#endif
#ifndef MCTS_ZT
#define MCTS_ZT 1        // no-move test as one 3-input LOP3 predicate on the two words
#endif
#ifndef MCTS_PRED_FLIP
#define MCTS_PRED_FLIP 1 // 32-bit ray flips: the kept run or-ed in by one predicated LOP3
#endif
#ifndef MCTS_FLIP_K
#define MCTS_FLIP_K 1    // flip carries from K = ~ray + first (saves the O | ~ray and 2 LOP3/direction)
#endif

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

// ---------------------------------------------------------------------------
// Plain rules (tree expansion, terminal tests, input generator).
// ---------------------------------------------------------------------------

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

// Uniform pick (R4): k = floor(r * c / 2^32), then the k-th legal
// square in ascending order.
__device__ __forceinline__ int pick_square(u64 moves, u32 r) {
  u32 c = (u32)__popcll(moves);
  return kth_set_bit(moves, __umulhi(r, c));
}

// Terminal test: neither side has a move.
__device__ __forceinline__ bool is_terminal(u64 P, u64 O, u64 legalP) {
  return legalP == 0ULL && legal_moves(O, P) == 0ULL;
}

// ---------------------------------------------------------------------------
// Counter-based RNG (R5).
// ---------------------------------------------------------------------------

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

// Stream of RNG words for one playout: word w is output[w % 4] of
// Philox(counter = (c0, c1, c2, w / 4), key = seed); the unread words of the
// current block are kept as a queue.
struct PlayoutRng {
  uint2 key;
  u32 c0, c1, c2;
  u32 w;
  uint4 buf;
  __device__ __forceinline__ u32 next() {
    if ((w & 3u) == 0u) buf = philox4x32_10(make_uint4(c0, c1, c2, w >> 2), key);
    ++w;
    const u32 r = buf.x;
    buf.x = buf.y;
    buf.y = buf.z;
    buf.z = buf.w;
    return r;
  }
  // The same stream with the word index kept by the caller (the playout's
  // ply counter: one word per non-pass decision, so w == plies so far).
  __device__ __forceinline__ u32 next_at(u32 n) {
    if ((n & 3u) == 0u) buf = philox4x32_10(make_uint4(c0, c1, c2, n >> 2), key);
    const u32 r = buf.x;
    buf.x = buf.y;
    buf.y = buf.z;
    buf.z = buf.w;
    return r;
  }
};

// ---------------------------------------------------------------------------
// Hot ply loop.
// ---------------------------------------------------------------------------

// Powers of two in constant memory: as IMAD multipliers they keep shifts and
// adds on the FMA pipe (ptxas cannot fold them back into ALU-pipe SHF/IADD3).
__constant__ u32 c_pow2[33] = {
    1u, 2u, 4u, 8u, 16u, 32u, 64u, 128u, 256u, 512u, 1024u, 2048u, 4096u, 8192u, 16384u, 32768u,
    1u << 16, 1u << 17, 1u << 18, 1u << 19, 1u << 20, 1u << 21, 1u << 22, 1u << 23, 1u << 24,
    1u << 25, 1u << 26, 1u << 27, 1u << 28, 1u << 29, 1u << 30, 1u << 31, 0u};

__device__ __forceinline__ u64 join32(u32 lo, u32 hi) { return ((u64)hi << 32) | lo; }
__device__ __forceinline__ u32 add_f(u32 a, u32 b) { return a * c_pow2[0] + b; }         // a + b
__device__ __forceinline__ u32 sub_f(u32 a, u32 b) { return b * (0u - c_pow2[0]) + a; }  // a - b

// Disjoint 64-bit or / subset and-not as two independent 32-bit IMADs:
// a | b when a & b == 0 (no carries), a & ~b when b is a subset of a (no borrows).
__device__ __forceinline__ u64 or_disjoint(u64 a, u64 b) {
#if MCTS_UPD_F
  return join32(add_f((u32)a, (u32)b), add_f((u32)(a >> 32), (u32)(b >> 32)));
#else
  return a | b;
#endif
}
__device__ __forceinline__ u64 andnot_subset(u64 a, u64 b) {
#if MCTS_UPD_F
  return join32(sub_f((u32)a, (u32)b), sub_f((u32)(a >> 32), (u32)(b >> 32)));
#else
  return a & ~b;
#endif
}

// Horizontal (+1) moves by carry propagation, per 32-bit half (a row never
// spans halves and no carry leaves a row: the landing square of a run ending
// on column 6 is column 7, and column 7 is never in M). t = P<<1 per half;
// s = M + t carries each adjacent opponent run to its landing square; s & ~t
// keeps the landings (plus non-carried O / P squares, removed by the caller's
// final empty-square mask).
__device__ __forceinline__ u64 east_moves(u64 P, u64 M) {
#if MCTS_EAST_F
  const u32 two = c_pow2[1];
  const u32 tl = (u32)P * two, th = (u32)(P >> 32) * two;
  const u32 sl = add_f((u32)M, tl), shh = add_f((u32)(M >> 32), th);
#else
  const u32 tl = (u32)P << 1, th = (u32)(P >> 32) << 1;
  const u32 sl = (u32)M + tl, shh = (u32)(M >> 32) + th;
#endif
  return join32(sl & ~tl, shh & ~th);
}

// One upward direction (+S, S in {7, 8, 9}) by a doubled-propagator fill: two
// single steps cover a 2-disc run, two double steps (M2 = M & M<<S) extend it
// to the 6-disc maximum. Left shifts only (MCTS_SPLIT = 0 path).
template <int S>
__device__ __forceinline__ u64 up_moves(u64 P, u64 M) {
  const u64 M2 = M & (M << S);
  u64 t = M & (P << S);
  t |= M & (t << S);
  t |= M2 & (t << (2 * S));
  t |= M2 & (t << (2 * S));
  return t << S;
}

// The same direction on 32-bit halves (rows 0-3 in lo, rows 4-7 in hi). An
// upward run only ever moves from lo into hi, so lo is filled on its own
// (three steps reach row 3 from row 0), then its top row crosses into hi once
// — with P's top row, as the seed of the hi fill (three steps reach row 6 from
// row 4) — instead of a funnel shift at every step of a 64-bit fill. All
// left shifts are IMADs by 2^S (FMA pipe); the two cross terms are the only
// shifts left on the ALU pipe. The landing squares t << S are or-ed into
// (ml, mh).
// One LOP3 with a fixed truth table (a = 0xF0, b = 0xCC, c = 0xAA). Written as
// PTX so ptxas keeps the shared masks M in registers instead of re-fusing
// O & kInner into every step (which costs a second LOP3 per step).
template <u32 LUT>
__device__ __forceinline__ u32 lop3(u32 a, u32 b, u32 c) {
  u32 r;
  asm("lop3.b32 %0, %1, %2, %3, %4;" : "=r"(r) : "r"(a), "r"(b), "r"(c), "n"(LUT));
  return r;
}
constexpr u32 kOrAnd = 0xF8;  // a | (b & c)
constexpr u32 kAndOr = 0xA8;  // (a | b) & c

template <int S>
__device__ __forceinline__ void up_moves_split(u32 Pl, u32 Ph, u32 Ml, u32 Mh, u32& ml, u32& mh) {
  const u32 p = c_pow2[S];
  u32 tl = Ml & (Pl * p);
  tl = lop3<kOrAnd>(tl, Ml, tl * p);
  tl = lop3<kOrAnd>(tl, Ml, tl * p);
  const u32 xt = tl >> (32 - S);
  const u32 pf = (u32)((join32(Pl, Ph) << S) >> 32);  // one funnel SHF: Ph << S | Pl >> (32 - S)
  u32 th = lop3<kAndOr>(pf, xt, Mh);
  th = lop3<kOrAnd>(th, Mh, th * p);
  th = lop3<kOrAnd>(th, Mh, th * p);
  ml |= tl * p;
  mh |= th * p + xt;
}

// Legal moves. The four upward directions (+1 by carries, +7/+8/+9 by fills)
// run on the board; the four downward ones run as upward directions of the
// bit-reversed board rP/rO (square s -> 63 - s is the 180-degree rotation, so
// -1/-7/-8/-9 become +1/+7/+8/+9 and the file masks are unchanged). The caller
// reuses rP/rO for the flips.
__device__ __forceinline__ u64 legal_moves_hot(u64 P, u64 O, u64 rP, u64 rO) {
#if MCTS_RM_BREV
  const u64 M = O & kInner, rM = __brevll(M);  // kInner is symmetric under bit reversal
#else
  const u64 M = O & kInner, rM = rO & kInner;
#endif
#if MCTS_SPLIT
  const u64 e = east_moves(P, M), re = east_moves(rP, rM);
  u32 ml = (u32)e, mh = (u32)(e >> 32), rl = (u32)re, rh = (u32)(re >> 32);
  up_moves_split<8>((u32)P, (u32)(P >> 32), (u32)O, (u32)(O >> 32), ml, mh);
  up_moves_split<7>((u32)P, (u32)(P >> 32), (u32)M, (u32)(M >> 32), ml, mh);
  up_moves_split<9>((u32)P, (u32)(P >> 32), (u32)M, (u32)(M >> 32), ml, mh);
  up_moves_split<8>((u32)rP, (u32)(rP >> 32), (u32)rO, (u32)(rO >> 32), rl, rh);
  up_moves_split<7>((u32)rP, (u32)(rP >> 32), (u32)rM, (u32)(rM >> 32), rl, rh);
  up_moves_split<9>((u32)rP, (u32)(rP >> 32), (u32)rM, (u32)(rM >> 32), rl, rh);
  return (join32(ml, mh) | __brevll(join32(rl, rh))) & ~(P | O);
#else
  u64 m = east_moves(P, M);
  m |= up_moves<8>(P, O);
  m |= up_moves<7>(P, M);
  m |= up_moves<9>(P, M);
  u64 r = east_moves(rP, rM);
  r |= up_moves<8>(rP, rO);
  r |= up_moves<7>(rP, rM);
  r |= up_moves<9>(rP, rM);
  return (m | __brevll(r)) & ~(P | O);
#endif
}

// Upward ray masks (squares strictly beyond sq in direction +1, +8, +7, +9 up
// to the board edge).
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

// Per-CTA shared table (u64 words): [0,256) ray masks rays[d*64 + sq],
// [256,512) the carry addend of the ray (K = ~ray + first square, mod 2^64;
// the first square alone when MCTS_FLIP_K = 0), [512,768) a byte-select LUT:
// byte (k*256 + b) = index of the k-th set bit of the byte b; [768,832) the
// square bits 1 << sq (one LDS instead of two ALU-pipe shifts per ply).
constexpr int kRayTable = 832;

// Build the table (into global memory once per handle; CTAs copy it).
__device__ __forceinline__ void fill_rays(u64* rays) {
  for (int i = threadIdx.x; i < 256; i += blockDim.x) {
    const u64 m = ray_mask(i >> 6, i & 63);
    rays[i] = m;
#if MCTS_FLIP_K
    rays[256 + i] = ~m + (m & (0ULL - m));
#else
    rays[256 + i] = m & (0ULL - m);
#endif
    u64 packed = 0;  // LUT bytes 8i .. 8i+7
    for (int j = 0; j < 8; ++j) {
      const int e = 8 * i + j, k = e >> 8, b = e & 255;
      int seen = 0, pos = 0;
      for (int q = 0; q < 8; ++q)
        if ((b >> q) & 1) { if (seen == k) { pos = q; break; } ++seen; }
      packed |= (u64)pos << (8 * j);
    }
    rays[512 + i] = packed;
    if (i < 64) rays[768 + i] = 1ULL << i;
  }
}

// Flips along an upward ray m by carry propagation: adding the ray's first
// square to (O | ~m) carries through the contiguous opponent run (and through
// the non-ray bits, all ones) and lands on the first non-opponent ray square.
// run = ray squares that carried (~s & O & m); kept iff the landing square
// s & m & P is non-empty. With MCTS_FLIP_K the sum is formed as (O & m) + K,
// K = ~m + first (O & m and ~m share no bits, so O | ~m = (O & m) + ~m): one
// LOP3 per half for O & m, and the run update f | (~s & Om) is one 3-input
// LOP3 per half.
__device__ __forceinline__ void up_flips(u64& f, u64 k, u64 P, u64 O, u64 m) {
#if MCTS_FLIP_K
  const u64 Om = O & m;
  const u64 s = Om + k;
  if (s & m & P) f |= ~s & Om;
#else
  const u64 s = (O | ~m) + k;
  if (s & m & P) f |= ~s & O & m;
#endif
}

// All 8 directions: the 4 upward ones on the board, the 4 downward ones as
// upward rays of square 63 - sq on the bit-reversed board rP/rO.
__device__ __forceinline__ u64 flips_hot(int sq, u64 P, u64 O, u64 rP, u64 rO,
                                         const u64* __restrict__ rays) {
  u64 f = 0;
  up_flips(f, rays[256 + sq], P, O, rays[sq]);
  up_flips(f, rays[320 + sq], P, O, rays[64 + sq]);
  up_flips(f, rays[384 + sq], P, O, rays[128 + sq]);
  up_flips(f, rays[448 + sq], P, O, rays[192 + sq]);
  const int rs = 63 - sq;
  u64 g = 0;
  up_flips(g, rays[256 + rs], rP, rO, rays[rs]);
  up_flips(g, rays[320 + rs], rP, rO, rays[64 + rs]);
  up_flips(g, rays[384 + rs], rP, rO, rays[128 + rs]);
  up_flips(g, rays[448 + rs], rP, rO, rays[192 + rs]);
  return f | __brevll(g);
}

// One upward ray that lies inside a single 32-bit word (k = that word of K).
// The 64-bit carry never leaves the ray's word, so the sum is a 32-bit add.
__device__ __forceinline__ void up_flips32(u32& f, u32 k, u32 P, u32 O, u32 m) {
  const u32 Om = O & m;
  const u32 s = add_f(Om, k);
#if MCTS_PRED_FLIP == 2
  // no select: h = umulhi(L, 2^32 - 1) = L ? L - 1 : 0 for the landing bit L,
  // and the kept run is ~s & m & h (the carried squares below L on the ray)
  const u32 h = __umulhi(s & m & P, 0xFFFFFFFFu);
  f |= ~s & m & h;
#elif MCTS_PRED_FLIP
  // f |= ~s & Om under the landing predicate as ONE predicated LOP3 (the C++
  // form compiles to run LOP3 + SEL + a share of an OR-merge LOP3).
  asm("{\n\t.reg .pred p;\n\t.reg .b32 t;\n\t"
      "lop3.b32 t, %1, %2, %3, 0x80;\n\t"   // s & m & P: the landing square
      "setp.ne.u32 p, t, 0;\n\t"
      "@p lop3.b32 %0, %0, %1, %4, 0xF2;\n\t"  // f | (~s & Om)
      "}"
      : "+r"(f) : "r"(s), "r"(m), "r"(P), "r"(Om));
#else
  if (s & m & P) f |= ~s & Om;
#endif
}

// flips_hot with the rays split by half: of the two frames (board at sq, reversed
// board at 63 - sq) exactly one puts the move in the hi word, and all four
// upward rays from a hi-word square stay in the hi word (32-bit ops); the
// other frame's square is in the lo word, where the +1 ray stays in the lo
// word and only the +8/+7/+9 rays need 64-bit carries. The frames are chosen
// per lane with selects (no divergence) and the result mapped back to the board.
__device__ __forceinline__ u64 flips_hot_xy(int sq, u64 P, u64 O, u64 rP, u64 rO,
                                            const u64* __restrict__ rays, bool hx) {
  const int xs = hx ? sq : 63 - sq, ys = 63 - xs;
  const u32 XP = hx ? (u32)(P >> 32) : (u32)(rP >> 32);
  const u32 XO = hx ? (u32)(O >> 32) : (u32)(rO >> 32);
  const u64 YP = hx ? rP : P, YO = hx ? rO : O;
  const u32* r32 = reinterpret_cast<const u32*>(rays);
  u32 fx = 0;
  up_flips32(fx, r32[2 * (256 + xs) + 1], XP, XO, r32[2 * xs + 1]);
  up_flips32(fx, r32[2 * (320 + xs) + 1], XP, XO, r32[2 * (64 + xs) + 1]);
  up_flips32(fx, r32[2 * (384 + xs) + 1], XP, XO, r32[2 * (128 + xs) + 1]);
  up_flips32(fx, r32[2 * (448 + xs) + 1], XP, XO, r32[2 * (192 + xs) + 1]);
  u32 fe = 0;
  up_flips32(fe, r32[2 * (256 + ys)], (u32)YP, (u32)YO, r32[2 * ys]);
  u64 fy = fe;
  up_flips(fy, rays[320 + ys], YP, YO, rays[64 + ys]);
  up_flips(fy, rays[384 + ys], YP, YO, rays[128 + ys]);
  up_flips(fy, rays[448 + ys], YP, YO, rays[192 + ys]);
  // Back to board coordinates: f = v | brev(u), u the reversed frame's flips
  // and v the board frame's (brev maps word w of one frame to word 1-w).
#if MCTS_MAPBACK3
  // hx: f = (fx << 32) | brev(fy); else f = fy | brev(fx << 32) = fy | brev(fx)
  const u32 ylo = (u32)fy, yhi = (u32)(fy >> 32);
  const u32 lo = hx ? __brev(yhi) : (ylo | __brev(fx));
  const u32 hi = hx ? (fx | __brev(ylo)) : yhi;
  return join32(lo, hi);
#else
  const u64 u = hx ? fy : join32(0u, fx);
  const u64 v = hx ? join32(0u, fx) : fy;
  return v | __brevll(u);
#endif
}

// The flips the ply loop uses (and the device perft pins).
__device__ __forceinline__ u64 flips_loop(int sq, u64 P, u64 O, u64 rP, u64 rO,
                                          const u64* __restrict__ rays) {
#if MCTS_FLIP_XY
  return flips_hot_xy(sq, P, O, rP, rO, rays, sq >= 32);
#else
  return flips_hot(sq, P, O, rP, rO, rays);
#endif
}

// k-th set bit: three popc levels down to a byte, then the byte-select LUT.
__device__ __forceinline__ int kth_set_bit_lut(u64 m, u32 k, const unsigned char* __restrict__ lut,
                                               bool* in_hi = nullptr) {
  u32 lo = (u32)m, hi = (u32)(m >> 32);
  u32 c = __popc(lo);
  bool up = k >= c;
  if (in_hi) *in_hi = up;  // the square is >= 32
  u32 x = up ? hi : lo;
  k -= up ? c : 0u;
  int base = up ? 32 : 0;
#if MCTS_PICK_SHL
  c = __popc(x * c_pow2[16]); up = k >= c; x = up ? (x >> 16) : x; k -= up ? c : 0u; base += up ? 16 : 0;
  c = __popc(x * c_pow2[24]); up = k >= c; x = up ? (x >> 8) : x;  k -= up ? c : 0u; base += up ? 8 : 0;
#else
  c = __popc(x & 0xFFFFu); up = k >= c; x = up ? (x >> 16) : x; k -= up ? c : 0u; base += up ? 16 : 0;
  c = __popc(x & 0xFFu);   up = k >= c; x = up ? (x >> 8) : x;  k -= up ? c : 0u; base += up ? 8 : 0;
#endif
  return base + lut[(k << 8) | (x & 0xFFu)];
}

// One decision for the side owning P: returns false if P has no move (a pass;
// nothing changes, no RNG word consumed), else plays the uniformly random move.
__device__ __forceinline__ bool ply(u64& P, u64& O, PlayoutRng& rng, u32 n, const u64* __restrict__ rays) {
  const u64 rP = __brevll(P), rO = __brevll(O);
  const u64 moves = legal_moves_hot(P, O, rP, rO);
#if MCTS_ZT
  if (((u32)moves | (u32)(moves >> 32)) == 0u) return false;
#else
  if (moves == 0ULL) return false;
#endif
#if MCTS_NW
  const u32 k = __umulhi(rng.next_at(n), (u32)__popcll(moves));
#else
  const u32 k = __umulhi(rng.next(), (u32)__popcll(moves));
#endif
#if MCTS_PICK_LUT && MCTS_FLIP_XY && MCTS_HXP
  bool hx;  // the pick's first level already decided the half: the flips' frame
  const int sq = kth_set_bit_lut(moves, k, reinterpret_cast<const unsigned char*>(rays + 512), &hx);
  const u64 f = flips_hot_xy(sq, P, O, rP, rO, rays, hx);
#else
#if MCTS_PICK_LUT
  const int sq = kth_set_bit_lut(moves, k, reinterpret_cast<const unsigned char*>(rays + 512));
#else
  const int sq = kth_set_bit(moves, k);
#endif
  const u64 f = flips_loop(sq, P, O, rP, rO, rays);
#endif
#if MCTS_BIT_LUT
  P = or_disjoint(P, or_disjoint(f, rays[768 + sq]));
#else
  P = or_disjoint(P, or_disjoint(f, 1ULL << sq));
#endif
  O = andnot_subset(O, f);
  return true;
}

// One random playout from (me to move, op). Returns +1 / 0 / -1 for the side
// to move at the start (R3), adds the non-pass plies to *plies.
// Two consecutive passes end the game. Unrolled by two so each side keeps its
// registers (no swaps).
__device__ __forceinline__ int playout(u64 me, u64 op, uint2 key, u32 c0, u32 c1, u32 c2,
                                       const u64* __restrict__ rays, u32* plies) {
  PlayoutRng rng;
  rng.key = key; rng.c0 = c0; rng.c1 = c1; rng.c2 = c2; rng.w = 0;
  rng.buf = make_uint4(0, 0, 0, 0);
  bool passed = false;
  u32 n = 0;
  // Every move fills one empty square, so the board is full (neither side can
  // move: game over) exactly when n reaches the starting number of empties;
  // testing that skips the two move generations that would establish it at the
  // end of most random games.
  const u32 empties = 64u - (u32)__popcll(me | op);
  for (;;) {
    if (n == empties) break;
    if (ply(me, op, rng, n, rays)) { passed = false; ++n; }
    else if (passed) break;
    else passed = true;
    if (n == empties) break;
    if (ply(op, me, rng, n, rays)) { passed = false; ++n; }
    else if (passed) break;
    else passed = true;
  }
  *plies += n;
  const int a = __popcll(me), b = __popcll(op);
  return (a > b) - (a < b);
}


// ---------------------------------------------------------------------------
// Two playouts per thread (MCTS_PAIR tuning variant): playouts X
// and Y advance in lock step, one ply each per half-step, so the compiler can
// interleave their independent instruction streams. Each half-step is one
// branch-free block (movegen, pick, flips and a board update masked by "has a
// move", as IMADs by 0/1) preceded by the rare Philox refills and followed by
// the pass / game-end bookkeeping; a finished playout keeps computing on an
// empty move mask and changes nothing. Same RNG words, same moves, same
// results as playout() for each of the two.
// ---------------------------------------------------------------------------
struct PairSide {
  u32 n, empties, c0, c2;
  uint4 buf;
  bool fresh, passed, done;
};

__device__ __forceinline__ void pair_init(PairSide& X, u64 me, u64 op, u32 c0, u32 c2, bool act) {
  X.n = 0;
  X.empties = 64u - (u32)__popcll(me | op);
  X.c0 = c0;
  X.c2 = c2;
  X.buf = make_uint4(0, 0, 0, 0);
  X.fresh = false;
  X.passed = false;
  X.done = !act || X.empties == 0u;
}

__device__ __forceinline__ void pair_refill(PairSide& X, uint2 key, u32 c1) {
  if (!X.done && (X.n & 3u) == 0u && !X.fresh) {
    X.buf = philox4x32_10(make_uint4(X.c0, c1, X.c2, X.n >> 2), key);
    X.fresh = true;
  }
}

// The branch-free part of one decision for the side owning P: returns whether
// a move was played (P, O updated).
__device__ __forceinline__ bool pair_ply(u64& P, u64& O, const PairSide& X, const u64* __restrict__ rays) {
  const u64 rP = __brevll(P), rO = __brevll(O);
  u64 moves = legal_moves_hot(P, O, rP, rO);
  moves = X.done ? 0ULL : moves;
  const bool has = ((u32)moves | (u32)(moves >> 32)) != 0u;
  const u32 k = __umulhi(X.buf.x, (u32)__popcll(moves));
  bool hx;
  const int sq = kth_set_bit_lut(moves, k, reinterpret_cast<const unsigned char*>(rays + 512), &hx);
  const u64 f = flips_hot_xy(sq, P, O, rP, rO, rays, hx);
  const u32 h = has ? 1u : 0u;
  const u64 add = or_disjoint(f, rays[768 + sq]);
  P = join32((u32)add * h + (u32)P, (u32)(add >> 32) * h + (u32)(P >> 32));
  O = join32((u32)f * (0u - h) + (u32)O, (u32)(f >> 32) * (0u - h) + (u32)(O >> 32));
  return has;
}

__device__ __forceinline__ void pair_book(PairSide& X, bool has) {
  if (has) {
    ++X.n;
    X.passed = false;
    X.fresh = false;
    X.buf.x = X.buf.y;
    X.buf.y = X.buf.z;
    X.buf.z = X.buf.w;
    if (X.n == X.empties) X.done = true;
  } else if (!X.done) {
    if (X.passed) X.done = true;
    else X.passed = true;
  }
}

// Returns the two results (+1 / 0 / -1 for each start position's side to
// move; an inactive side returns 0) and adds both ply counts to *plies.
__device__ __forceinline__ void playout_pair(u64 meX, u64 opX, u32 c0X, u32 c2X, bool actX,
                                             u64 meY, u64 opY, u32 c0Y, u32 c2Y, bool actY,
                                             uint2 key, u32 c1, const u64* __restrict__ rays,
                                             u32* plies, int& rX, int& rY) {
  PairSide X, Y;
  pair_init(X, meX, opX, c0X, c2X, actX);
  pair_init(Y, meY, opY, c0Y, c2Y, actY);
  while (!(X.done && Y.done)) {
    pair_refill(X, key, c1);
    pair_refill(Y, key, c1);
    const bool hx1 = pair_ply(meX, opX, X, rays);
    const bool hy1 = pair_ply(meY, opY, Y, rays);
    pair_book(X, hx1);
    pair_book(Y, hy1);
    if (X.done && Y.done) break;
    pair_refill(X, key, c1);
    pair_refill(Y, key, c1);
    const bool hx2 = pair_ply(opX, meX, X, rays);
    const bool hy2 = pair_ply(opY, meY, Y, rays);
    pair_book(X, hx2);
    pair_book(Y, hy2);
  }
  *plies += X.n + Y.n;
  const int a = __popcll(meX), b = __popcll(opX), c = __popcll(meY), d = __popcll(opY);
  rX = actX ? (a > b) - (a < b) : 0;
  rY = actY ? (c > d) - (c < d) : 0;
}

}  // namespace mcts_dev
