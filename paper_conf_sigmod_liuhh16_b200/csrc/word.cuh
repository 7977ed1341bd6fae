// word.cuh -- the per-vertex status word of a group: one bit per BFS instance.
//
// PAPER.md §6: the Bitwise Status Array keeps, per vertex, the statuses
// of all instances of a group "in a single variable": 1 = visited, 0 = not.  The paper
// packs 32..128 instances with int / int4 / long4 vector types and
// defaults to 128.  Here: uint32_t (W = 32), u64 (W = 64) and a
// 16-byte aligned pair of u64 (W = 128) moved with one 128-bit load/store.
// Bit j of the word is instance j of the group (BFS-j); the 32-bit piece k of a word is
// bits [32k, 32k + 32) (little-endian), which is what the depth recorder iterates.
#pragma once
#include <cstdint>

namespace ibfs {

struct __align__(16) u128 {
  unsigned long long lo, hi;
};

// ---- bitwise algebra ---------------------------------------------------------------
__host__ __device__ __forceinline__ uint32_t wand(uint32_t a, uint32_t b) { return a & b; }
__host__ __device__ __forceinline__ unsigned long long wand(unsigned long long a, unsigned long long b) { return a & b; }
__host__ __device__ __forceinline__ u128 wand(u128 a, u128 b) { return {a.lo & b.lo, a.hi & b.hi}; }

__host__ __device__ __forceinline__ uint32_t wor(uint32_t a, uint32_t b) { return a | b; }
__host__ __device__ __forceinline__ unsigned long long wor(unsigned long long a, unsigned long long b) { return a | b; }
__host__ __device__ __forceinline__ u128 wor(u128 a, u128 b) { return {a.lo | b.lo, a.hi | b.hi}; }

// a & ~b
__host__ __device__ __forceinline__ uint32_t wandn(uint32_t a, uint32_t b) { return a & ~b; }
__host__ __device__ __forceinline__ unsigned long long wandn(unsigned long long a, unsigned long long b) { return a & ~b; }
__host__ __device__ __forceinline__ u128 wandn(u128 a, u128 b) { return {a.lo & ~b.lo, a.hi & ~b.hi}; }

__host__ __device__ __forceinline__ uint32_t wnot(uint32_t a) { return ~a; }
__host__ __device__ __forceinline__ unsigned long long wnot(unsigned long long a) { return ~a; }
__host__ __device__ __forceinline__ u128 wnot(u128 a) { return {~a.lo, ~a.hi}; }

__host__ __device__ __forceinline__ bool wzero(uint32_t a) { return a == 0; }
__host__ __device__ __forceinline__ bool wzero(unsigned long long a) { return a == 0; }
__host__ __device__ __forceinline__ bool wzero(u128 a) { return (a.lo | a.hi) == 0; }

__host__ __device__ __forceinline__ bool weq(uint32_t a, uint32_t b) { return a == b; }
__host__ __device__ __forceinline__ bool weq(unsigned long long a, unsigned long long b) { return a == b; }
__host__ __device__ __forceinline__ bool weq(u128 a, u128 b) { return a.lo == b.lo && a.hi == b.hi; }

template <typename T> __host__ __device__ __forceinline__ T wzero_value() { return T{}; }
template <> __host__ __device__ __forceinline__ u128 wzero_value<u128>() { return {0ull, 0ull}; }

__device__ __forceinline__ int wpopc(uint32_t a) { return __popc(a); }
__device__ __forceinline__ int wpopc(unsigned long long a) { return __popcll(a); }
__device__ __forceinline__ int wpopc(u128 a) { return __popcll(a.lo) + __popcll(a.hi); }

template <typename T> struct WordBits;
template <> struct WordBits<uint32_t> { static constexpr int value = 32; };
template <> struct WordBits<unsigned long long> { static constexpr int value = 64; };
template <> struct WordBits<u128> { static constexpr int value = 128; };

// 32-bit piece k (k < W/32)
__device__ __forceinline__ uint32_t wpiece(uint32_t a, int) { return a; }
__device__ __forceinline__ uint32_t wpiece(unsigned long long a, int k) { return (uint32_t)(a >> (32 * k)); }
__device__ __forceinline__ uint32_t wpiece(u128 a, int k) {
  unsigned long long h = (k < 2) ? a.lo : a.hi;
  return (uint32_t)(h >> (32 * (k & 1)));
}

// word from its 32-bit pieces (little-endian)
template <typename T> __device__ __forceinline__ T wfrom_pieces(const uint32_t *p);
template <> __device__ __forceinline__ uint32_t wfrom_pieces<uint32_t>(const uint32_t *p) { return p[0]; }
template <> __device__ __forceinline__ unsigned long long wfrom_pieces<unsigned long long>(const uint32_t *p) {
  return ((unsigned long long)p[1] << 32) | p[0];
}
template <> __device__ __forceinline__ u128 wfrom_pieces<u128>(const uint32_t *p) {
  return {((unsigned long long)p[1] << 32) | p[0], ((unsigned long long)p[3] << 32) | p[2]};
}

// Bits [h * W/2, (h + 1) * W/2) of a word, h in {0, 1}, right-aligned.
__device__ __forceinline__ unsigned long long whalf(uint32_t a, int h) { return h ? (a >> 16) : (a & 0xffffu); }
__device__ __forceinline__ unsigned long long whalf(unsigned long long a, int h) {
  return h ? (a >> 32) : (a & 0xffffffffull);
}
__device__ __forceinline__ unsigned long long whalf(u128 a, int h) { return h ? a.hi : a.lo; }

// word with the low `n` bits set (n <= W): the real instances of a (possibly short) group
template <typename T> __host__ __device__ __forceinline__ T wlowmask(int n);
template <> __host__ __device__ __forceinline__ uint32_t wlowmask<uint32_t>(int n) {
  return n >= 32 ? 0xffffffffu : ((1u << n) - 1u);
}
template <> __host__ __device__ __forceinline__ unsigned long long wlowmask<unsigned long long>(int n) {
  return n >= 64 ? ~0ull : ((1ull << n) - 1ull);
}
template <> __host__ __device__ __forceinline__ u128 wlowmask<u128>(int n) {
  u128 r;
  r.lo = n >= 64 ? ~0ull : ((1ull << n) - 1ull);
  r.hi = n >= 128 ? ~0ull : (n <= 64 ? 0ull : ((1ull << (n - 64)) - 1ull));
  return r;
}

// ---- memory ---------------------------------------------------------------------------
// Read-only-in-this-kernel loads go through the non-coherent path.
__device__ __forceinline__ uint32_t ldg(const uint32_t *p) { return __ldg(p); }
__device__ __forceinline__ unsigned long long ldg(const unsigned long long *p) { return __ldg(p); }
__device__ __forceinline__ u128 ldg(const u128 *p) {
  ulonglong2 v = __ldg(reinterpret_cast<const ulonglong2 *>(p));
  return {v.x, v.y};
}

// Coherent loads (data another CTA of this launch may have written atomically).
__device__ __forceinline__ uint32_t ldv(const uint32_t *p) { return *(const volatile uint32_t *)p; }
__device__ __forceinline__ unsigned long long ldv(const unsigned long long *p) {
  return *(const volatile unsigned long long *)p;
}
__device__ __forceinline__ u128 ldv(const u128 *p) {
  const volatile unsigned long long *q = (const volatile unsigned long long *)p;
  return {q[0], q[1]};
}

// L2-coherent loads (ld.global.cg: skip L1) of words another CTA of this launch wrote
// before a grid barrier.
__device__ __forceinline__ uint32_t ldcg(const uint32_t *p) { return __ldcg(p); }
__device__ __forceinline__ uint32_t ldcg_w(const uint32_t *p) { return __ldcg(p); }
__device__ __forceinline__ unsigned long long ldcg_w(const unsigned long long *p) { return __ldcg(p); }
__device__ __forceinline__ u128 ldcg_w(const u128 *p) {
  ulonglong2 v = __ldcg(reinterpret_cast<const ulonglong2 *>(p));
  return {v.x, v.y};
}

__device__ __forceinline__ uint32_t ld(const uint32_t *p) { return *p; }
__device__ __forceinline__ unsigned long long ld(const unsigned long long *p) { return *p; }
__device__ __forceinline__ u128 ld(const u128 *p) {
  ulonglong2 v = *reinterpret_cast<const ulonglong2 *>(p);
  return {v.x, v.y};
}
__device__ __forceinline__ void st(uint32_t *p, uint32_t v) { *p = v; }
__device__ __forceinline__ void st(unsigned long long *p, unsigned long long v) { *p = v; }
__device__ __forceinline__ void st(u128 *p, u128 v) {
  *reinterpret_cast<ulonglong2 *>(p) = make_ulonglong2(v.lo, v.hi);
}
// streaming (evict-first) stores: words no kernel of this batch reads again
__device__ __forceinline__ void st_cs(uint32_t *p, uint32_t v) { __stcs(p, v); }
__device__ __forceinline__ void st_cs(unsigned long long *p, unsigned long long v) { __stcs(p, v); }
__device__ __forceinline__ void st_cs(u128 *p, u128 v) {
  __stcs(reinterpret_cast<ulonglong2 *>(p), make_ulonglong2(v.lo, v.hi));
}

// Atomic OR without return (compiles to RED.OR).  No 128-bit atomicOr exists, so W = 128
// issues two independent 64-bit reductions; OR is bitwise, so the halves commute
// (reading #10).  Zero halves are skipped.
__device__ __forceinline__ void red_or(uint32_t *p, uint32_t v) { atomicOr(p, v); }
__device__ __forceinline__ void red_or(unsigned long long *p, unsigned long long v) { atomicOr(p, v); }
__device__ __forceinline__ void red_or(u128 *p, u128 v) {
  unsigned long long *q = reinterpret_cast<unsigned long long *>(p);
  if (v.lo) atomicOr(q, v.lo);
  if (v.hi) atomicOr(q + 1, v.hi);
}

// Set bit j of the word at p (atomic on its 32-bit piece).
template <typename T> __device__ __forceinline__ void set_bit_atomic(T *p, int j) {
  atomicOr(reinterpret_cast<uint32_t *>(p) + (j >> 5), 1u << (j & 31));
}

// Warp OR-reduce of a word (every lane gets the result).
__device__ __forceinline__ uint32_t warp_or(uint32_t a) { return __reduce_or_sync(0xffffffffu, a); }
__device__ __forceinline__ unsigned long long warp_or(unsigned long long a) {
  uint32_t lo = __reduce_or_sync(0xffffffffu, (uint32_t)a);
  uint32_t hi = __reduce_or_sync(0xffffffffu, (uint32_t)(a >> 32));
  return ((unsigned long long)hi << 32) | lo;
}
__device__ __forceinline__ u128 warp_or(u128 a) { return {warp_or(a.lo), warp_or(a.hi)}; }

}  // namespace ibfs
