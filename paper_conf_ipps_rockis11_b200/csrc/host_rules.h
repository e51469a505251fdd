// host_rules.h — the game rules, RNG and playout on host threads, for the
// host-side parts of the library (the hybrid schemes: host_mcts.cpp,
// hosted.cpp). Same rules, Philox streams and pick as the device path
// (R3-R7); host code only ever runs NEXT TO a GPU search, never as a
// substitute for it.
#pragma once
#include <cstdint>

namespace host_rules {

typedef uint64_t u64;
typedef uint32_t u32;

constexpr u64 kInner = 0x7E7E7E7E7E7E7E7EULL;

template <int S>
inline u64 sh(u64 x) {
  if constexpr (S > 0) return x << S;
  else return x >> (-S);
}

template <int S>
inline u64 dir_moves(u64 P, u64 M) {
  u64 t = M & sh<S>(P);
  for (int i = 0; i < 5; ++i) t |= M & sh<S>(t);
  return sh<S>(t);
}

inline u64 legal(u64 P, u64 O) {
  const u64 M = O & kInner;
  u64 m = dir_moves<1>(P, M) | dir_moves<-1>(P, M) | dir_moves<8>(P, O) | dir_moves<-8>(P, O);
  m |= dir_moves<7>(P, M) | dir_moves<-7>(P, M) | dir_moves<9>(P, M) | dir_moves<-9>(P, M);
  return m & ~(P | O);
}

template <int S>
inline u64 dir_flips(u64 x, u64 P, u64 M) {
  u64 t = M & sh<S>(x);
  for (int i = 0; i < 5; ++i) t |= M & sh<S>(t);
  return (sh<S>(t) & P) ? t : 0ULL;
}

inline u64 flips(int sq, u64 P, u64 O) {
  const u64 x = 1ULL << sq, M = O & kInner;
  return dir_flips<1>(x, P, M) | dir_flips<-1>(x, P, M) | dir_flips<8>(x, P, O) |
         dir_flips<-8>(x, P, O) | dir_flips<7>(x, P, M) | dir_flips<-7>(x, P, M) |
         dir_flips<9>(x, P, M) | dir_flips<-9>(x, P, M);
}

inline int popc(u64 x) { return __builtin_popcountll(x); }

inline int kth_bit(u64 m, u32 k) {
  for (u32 i = 0; i < k; ++i) m &= m - 1;
  return __builtin_ctzll(m);
}

inline void philox(u32 c[4], u32 k0, u32 k1) {
  for (int i = 0; i < 10; ++i) {
    const u64 p0 = (u64)0xD2511F53u * c[0], p1 = (u64)0xCD9E8D57u * c[2];
    const u32 n0 = (u32)(p1 >> 32) ^ c[1] ^ k0, n2 = (u32)(p0 >> 32) ^ c[3] ^ k1;
    c[1] = (u32)p1;
    c[3] = (u32)p0;
    c[0] = n0;
    c[2] = n2;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
}

// One random playout; +1 / 0 / -1 for the side to move at the start.
inline int playout(u64 me, u64 op, u64 seed, u32 c0, u32 c1, u32 c2, u64* plies) {
  u32 buf[4] = {0, 0, 0, 0};
  u32 w = 0;
  bool start = true, passed = false;
  for (;;) {
    const u64 m = legal(me, op);
    if (m == 0) {
      if (passed) break;
      passed = true;
    } else {
      passed = false;
      if ((w & 3u) == 0u) {
        buf[0] = c0; buf[1] = c1; buf[2] = c2; buf[3] = w >> 2;
        philox(buf, (u32)seed, (u32)(seed >> 32));
      }
      const u32 r = buf[w & 3u];
      ++w;
      const int sq = kth_bit(m, (u32)(((u64)r * (u32)popc(m)) >> 32));
      const u64 f = flips(sq, me, op);
      me |= f | (1ULL << sq);
      op &= ~f;
      ++*plies;
    }
    const u64 t = me; me = op; op = t;
    start = !start;
  }
  const int a = popc(start ? me : op), b = popc(start ? op : me);
  return (a > b) - (a < b);
}

}  // namespace host_rules
