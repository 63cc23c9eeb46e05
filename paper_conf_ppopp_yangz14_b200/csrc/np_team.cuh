// np_team.cuh -- CUDA-NP master/slave team primitives for sm_100a.
//
// The paper (Yang & Zhou, PPoPP'14; "P:n" = line n of PAPER.md) turns every
// original thread into a *master* that owns S-1 *slaves* (S = slave_size
// counts the master).  Masters alone run sequential code
// (`if (slave_id==0)`, Fig 3b); at a parallel loop the whole team
// shares the iterations; live-ins reach the slaves through
// `read_from_master`; live-outs are combined by a reduction or
// a scan.  Two thread remaps:
//   intra-warp: the team is S consecutive lanes of one warp (shfl);
//   inter-warp: master = threadIdx.x, slave = threadIdx.y, so the team spans
//               S warps and talks through shared memory.
//
// This header holds those primitives written for sm_100a: `__shfl_*_sync`
// with a width argument (the Kepler `__shfl(var, lane, width)` of P:55),
// shared-memory exchange plus barriers for inter-warp teams, and the
// iteration distributions (cyclic = the paper's, block = the north star's).
// Nothing here depends on the oracle.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace cudanp {

constexpr unsigned kFull = 0xffffffffu;

enum Map : int { MAP_AUTO = 0, MAP_INTRA = 1, MAP_INTER = 2 };

// ---------------------------------------------------------------- launch overlap
// Programmatic dependent launch (sm_90+): the hot-path kernels are launched
// with programmatic stream serialization (launch_pdl in common.cuh), so the
// next kernel on the stream is scheduled while this one drains.  Every such
// kernel therefore waits for its predecessors' completion and memory
// (griddepcontrol.wait) before touching global memory -- reads and writes
// alike, so neither RAW nor WAR hazards can cross kernels -- and only then
// lets its own dependent launch (one kernel ahead at most).  Launched
// without the attribute both instructions are no-ops.
__device__ __forceinline__ void pdl_entry() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

enum Dist : int { DIST_CYCLIC = 0, DIST_BLOCK = 1 };

// ---------------------------------------------------------------- operators
struct OpSum {
  __device__ __forceinline__ static float apply(float a, float b) { return a + b; }
  // int32 sum wraps modulo 2^32 (R13): add in uint32.
  __device__ __forceinline__ static int32_t apply(int32_t a, int32_t b) {
    return (int32_t)((uint32_t)a + (uint32_t)b);
  }
  template <class T> __device__ __forceinline__ static T identity() { return T(0); }
};

struct OpMax {
  __device__ __forceinline__ static float apply(float a, float b) { return fmaxf(a, b); }
  __device__ __forceinline__ static int32_t apply(int32_t a, int32_t b) { return a > b ? a : b; }
  template <class T> __device__ __forceinline__ static T identity();
};
template <> __device__ __forceinline__ float OpMax::identity<float>() { return -__int_as_float(0x7f800000); }
template <> __device__ __forceinline__ int32_t OpMax::identity<int32_t>() { return INT32_MIN; }

// ---------------------------------------------------------------- vectors
template <class T> struct V4 { T x, y, z, w; };

// Streaming 128-bit load through the read-only path (LDG.E.128.CONSTANT).
// The asm stays `volatile`: a non-volatile asm with no memory operand counts
// as side-effect free, so the compiler may speculate it past the bound checks
// of the loop (an out-of-bounds load).  Load batching comes from the register
// budget given in __launch_bounds__, not from dropping volatile.
template <class T>
__device__ __forceinline__ V4<T> ldg4(const T* p) {
  V4<T> r;
  uint32_t a, b, c, d;
#if defined(CUDANP_L2_256B_ALL)
  asm volatile("ld.global.nc.L2::256B.v4.b32 {%0,%1,%2,%3}, [%4];"
#else
  asm volatile("ld.global.nc.v4.b32 {%0,%1,%2,%3}, [%4];"
#endif
               : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "l"(p));
  r.x = __builtin_bit_cast(T, a); r.y = __builtin_bit_cast(T, b);
  r.z = __builtin_bit_cast(T, c); r.w = __builtin_bit_cast(T, d);
  return r;
}
// Same with L1::no_allocate: data a warp touches once (TMV/MV matrix rows).
template <class T>
__device__ __forceinline__ V4<T> ldg4_stream(const T* p) {
  V4<T> r;
  uint32_t a, b, c, d;
#if defined(CUDANP_L2_256B)
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.b32 {%0,%1,%2,%3}, [%4];"
#else
  asm volatile("ld.global.nc.L1::no_allocate.v4.b32 {%0,%1,%2,%3}, [%4];"
#endif
               : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "l"(p));
  r.x = __builtin_bit_cast(T, a); r.y = __builtin_bit_cast(T, b);
  r.z = __builtin_bit_cast(T, c); r.w = __builtin_bit_cast(T, d);
  return r;
}
template <class T>
__device__ __forceinline__ T ldg1(const T* p) { return __ldg(p); }

// Bulk L2 prefetch through the TMA unit (cp.async.bulk.prefetch.L2, SASS
// UBLKPF.L2): fire-and-forget, no registers; 16-byte aligned, bytes % 16 == 0.
__device__ __forceinline__ void prefetch_l2(const void* p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// L2 prefetch of bytes [p, p + bytes).  It returns no data and the L2 is the
// device's point of coherence, so it may run BEFORE griddepcontrol.wait: a
// predecessor's later store to those bytes updates the L2 copy, and every load
// after the wait still sees it.  Latency-bound kernels use it to start their
// DRAM round trip while the predecessor drains (C1).  The copy
// engine does the work (one instruction per contiguous span, no load/store-unit
// replays); the span is widened to 16-byte boundaries, which never leaves the
// pages holding its first and last byte.
__device__ __forceinline__ void prefetch_l2_span(const void* p, int64_t bytes) {
  if (bytes <= 0) return;
  uintptr_t a = reinterpret_cast<uintptr_t>(p) & ~uintptr_t(15);
  const uintptr_t e = (reinterpret_cast<uintptr_t>(p) + (uintptr_t)bytes + 15) & ~uintptr_t(15);
  for (; a < e; a += 65536) {
    const uint32_t n = (uint32_t)(e - a < 65536 ? e - a : 65536);
    prefetch_l2(reinterpret_cast<const void*>(a), n);
  }
}

// Grid-wide L2 prefetch of rows [0, h) (each `row_bytes` long, row stride lda
// floats) of a row-major fp32 matrix and of the vector x[0, nx): CTA b takes
// its contiguous 1/gridDim of the rows (not the columns it reads itself), one
// row per lane of warp 0, so the whole grid pulls the operand in while it
// waits on its predecessor.
__device__ __forceinline__ void prefetch_l2_grid(const float* A, int64_t lda, int64_t h,
                                                 int64_t row_bytes, const float* x, int64_t nx) {
  const int tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  if (tid >= 32) return;
  const int64_t rpc = (h + gridDim.x - 1) / gridDim.x;
  const int64_t r0 = (int64_t)blockIdx.x * rpc, r1 = r0 + rpc < h ? r0 + rpc : h;
  if (lda * 4 == row_bytes) {  // dense rows: the CTA's rows are one span
    if (tid == 0 && r0 < r1) prefetch_l2_span(A + r0 * lda, (r1 - r0) * row_bytes);
  } else {
    for (int64_t r = r0 + tid; r < r1; r += 32) prefetch_l2_span(A + r * lda, row_bytes);
  }
  // x: CTA b takes the b-th 1/gridDim of it.
  const int64_t xpc = (nx + gridDim.x - 1) / gridDim.x;
  const int64_t x0 = (int64_t)blockIdx.x * xpc;
  if (tid == 1 && x0 < nx) prefetch_l2_span(x + x0, 4 * (x0 + xpc < nx ? xpc : nx - x0));
}

// 256-bit load (sm_100: LDG.E.ENL2.256.CONSTANT), 32-byte aligned: one
// request per lane covers a whole 32-byte sector, half the load instructions
// of 128-bit units for the same bytes in flight.
template <class T> struct V8 { T v[8]; };
template <class T>
__device__ __forceinline__ V8<T> ldg8(const T* p) {
  uint32_t a[8];
  asm volatile("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(a[0]), "=r"(a[1]), "=r"(a[2]), "=r"(a[3]), "=r"(a[4]), "=r"(a[5]), "=r"(a[6]),
                 "=r"(a[7])
               : "l"(p));
  V8<T> r;
#pragma unroll
  for (int k = 0; k < 8; ++k) r.v[k] = __builtin_bit_cast(T, a[k]);
  return r;
}

template <class T>
__device__ __forceinline__ void stg4(T* p, V4<T> v) {
  asm volatile("st.global.v4.b32 [%0], {%1,%2,%3,%4};" ::"l"(p),
               "r"(__builtin_bit_cast(uint32_t, v.x)), "r"(__builtin_bit_cast(uint32_t, v.y)),
               "r"(__builtin_bit_cast(uint32_t, v.z)), "r"(__builtin_bit_cast(uint32_t, v.w))
               : "memory");
}

// ---------------------------------------------------------------- distribution
// Iterations of a parallel loop of `n` units (a unit = V consecutive
// elements) owned by slave `s` of a team of S.
//  cyclic (P:166 `for(i=slave_id;i<N;i+=slave_size)`): s, s+S, ...
//  block  (north star; R5): chunk c = ceil(L/S) rounded up to a
//         multiple of V elements, i.e. cu = c/V units; [s*cu, min(n,(s+1)cu)).
// The bound check stays, so n may be any runtime value >= 0.
template <int S, int DIST>
struct Range {
  int64_t begin, end, step;
  __device__ __forceinline__ Range(int64_t n_units, int64_t n_elems, int V, int s) {
    if (DIST == DIST_CYCLIC) {
      begin = s; end = n_units; step = S;
    } else {
      int64_t c = (n_elems + S - 1) / S;
      int64_t cu = (c + V - 1) / V;
      begin = (int64_t)s * cu;
      end = begin + cu < n_units ? begin + cu : n_units;
      step = 1;
    }
  }
};

// ---------------------------------------------------------------- intra-warp team
// Team = S consecutive lanes (S a power of two <= 32).  slave =
// lane % S; the master is the team's lane 0; a warp holds 32/S teams
// (S=4 -> 8 masters + 24 slaves per warp).
template <int S>
struct IntraTeam {
  static_assert(S >= 1 && S <= 32 && (S & (S - 1)) == 0, "intra-warp S must be 2^k <= 32");
  static constexpr int kTeamsPerWarp = 32 / S;
  int lane, slave, team;  // team index within the warp

  __device__ __forceinline__ IntraTeam() {
    lane = threadIdx.x & 31;
    slave = lane & (S - 1);
    team = lane / S;
  }
  __device__ __forceinline__ bool is_master() const { return slave == 0; }

  // read_from_master: `__shfl(var, 0, slave_size)`.
  template <class T>
  __device__ __forceinline__ T read_from_master(T v) const {
    if (S == 1) return v;
    return __shfl_sync(kFull, v, 0, S);
  }
  // Value held by the team's last slave (scan carry).
  template <class T>
  __device__ __forceinline__ T from_last(T v) const {
    if (S == 1) return v;
    return __shfl_sync(kFull, v, S - 1, S);
  }
  // Reduction of the team's values (shfl for intra-warp NP):
  // butterfly over log2(S) steps; every team lane ends with the result.
  template <class Op, class T>
  __device__ __forceinline__ T reduce(T v) const {
#pragma unroll
    for (int o = S / 2; o > 0; o >>= 1) v = Op::apply(v, __shfl_xor_sync(kFull, v, o, S));
    return v;
  }
  // The same reduction through shared memory ("using shared memory";
  // the Fig 16 comparison): every lane writes its partial to the
  // warp's 32 slots and the master folds its team's S slots in slave order.
  // Only the master's return value is meaningful.
  template <class Op, class T>
  __device__ __forceinline__ T reduce_smem(T v, T* slots /*[32] per warp*/) const {
    slots[lane] = v;
    __syncwarp();
    T r = v;
    if (slave == 0) {
#pragma unroll
      for (int k = 1; k < S; ++k) r = Op::apply(r, slots[lane + k]);
    }
    __syncwarp();
    return r;
  }
  // Team mask for the width-S segment of this lane.
  __device__ __forceinline__ unsigned segment_mask() const {
    return S == 32 ? kFull : (((1u << S) - 1u) << (team * S));
  }
  // Inclusive scan over the team ("similar approach to the CUDA SDK"):
  // Hillis-Steele with shfl_up inside each width-S segment.
  template <class T>
  __device__ __forceinline__ T inclusive_scan(T v) const {
#pragma unroll
    for (int o = 1; o < S; o <<= 1) {
      T t = __shfl_up_sync(kFull, v, o, S);
      if (slave >= o) v = OpSum::apply(v, t);
    }
    return v;
  }
  // Exclusive value = inclusive value of the previous slave (0 for slave 0).
  template <class T>
  __device__ __forceinline__ T exclusive_from_inclusive(T incl) const {
    if (S == 1) return T(0);
    T t = __shfl_up_sync(kFull, incl, 1, S);
    return slave == 0 ? T(0) : t;
  }
};

// ---------------------------------------------------------------- redux.sync
// Hardware warp reductions (sm_80+ integer, sm_100a fp32 min/max) over a
// lane mask; segments of a width-S team each pass their own mask.
struct Redux {
  __device__ __forceinline__ static int32_t sum(int32_t v, unsigned mask) {
    return (int32_t)__reduce_add_sync(mask, (unsigned)v);
  }
  __device__ __forceinline__ static int32_t max(int32_t v, unsigned mask) {
    return __reduce_max_sync(mask, v);
  }
  __device__ __forceinline__ static float max(float v, unsigned mask) {
    float r;
    asm volatile("redux.sync.max.f32 %0, %1, %2;" : "=f"(r) : "f"(v), "r"(mask));
    return r;
  }
};

// ---------------------------------------------------------------- inter-warp team
// blockDim = (MX, S): master = threadIdx.x, slave = threadIdx.y.
// With MX = 32 masters a master's slaves sit in S different warps; the
// narrow-matrix TMV uses MX = 8 (4 slaves of 8 masters per warp, S <= 128).
// Every exchange goes through shared memory plus a CTA barrier (P:203,
// P:209).  All CTA threads must call the collective members (they contain
// __syncthreads).
template <int S>
struct InterTeam {
  static_assert(S >= 1 && S <= 128, "inter-warp S <= 128 (CTA = masters x S <= 1024 threads)");
  int master, slave;
  __device__ __forceinline__ InterTeam() {
    master = threadIdx.x;
    slave = threadIdx.y;
  }
  __device__ __forceinline__ bool is_master() const { return slave == 0; }

  // read_from_master through a per-master smem slot.
  template <class T>
  __device__ __forceinline__ T read_from_master(T v, T* slot /*[32]*/) const {
    if (S == 1) return v;
    if (slave == 0) slot[master] = v;
    __syncthreads();
    T r = slot[master];
    __syncthreads();
    return r;
  }
  // Two live-ins broadcast under one pair of barriers.
  template <class T>
  __device__ __forceinline__ void read_from_master(T& a, T& b, T* slot_a, T* slot_b) const {
    if (S == 1) return;
    if (slave == 0) { slot_a[master] = a; slot_b[master] = b; }
    __syncthreads();
    a = slot_a[master];
    b = slot_b[master];
    __syncthreads();
  }
};

// ---------------------------------------------------------------- multi-warp team
// S > 32 ("shared-memory fallback when S exceeds 32", north star): S/32
// consecutive warps of one CTA; shfl trees inside each warp and the
// warp results combined through shared memory.
template <int S>
struct MultiTeam {
  static_assert(S % 32 == 0 && S >= 64 && S <= 1024, "multi-warp teams: S = 64..1024");
  static constexpr int W = S / 32;  // warps per team
  int slave, team, lane, wit;       // wit: warp index inside the team
  __device__ __forceinline__ MultiTeam() {
    slave = threadIdx.x % S;
    team = threadIdx.x / S;
    lane = threadIdx.x & 31;
    wit = slave >> 5;
  }
  __device__ __forceinline__ bool is_master() const { return slave == 0; }

  // Reduction: shfl butterfly per warp, then the team's W warp results through
  // shared memory.  Every CTA thread must call it (it holds CTA barriers);
  // every team member returns the team's result.
  template <class Op, class T>
  __device__ __forceinline__ T reduce(T v, T* sm /*[teams*W]*/) const {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = Op::apply(v, __shfl_xor_sync(kFull, v, o));
    if (lane == 0) sm[team * W + wit] = v;
    __syncthreads();
    T r = sm[team * W];
#pragma unroll 4
    for (int k = 1; k < W; ++k) r = Op::apply(r, sm[team * W + k]);
    __syncthreads();
    return r;
  }
  // Exclusive scan over the S team threads (the sum of the lower slaves'
  // values); *total = the team's sum.  Inside a warp the exclusive value is
  // the previous lane's inclusive value (a shuffle), not incl - v, so fp32
  // prefixes carry no cancellation error.
  template <class T>
  __device__ __forceinline__ T exclusive_scan(T v, T* sm /*[teams*W]*/, T* total) const {
    T incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const T t = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl = OpSum::apply(incl, t);
    }
    const T prev = __shfl_up_sync(kFull, incl, 1);
    const T wexcl = lane == 0 ? T(0) : prev;
    if (lane == 31) sm[team * W + wit] = incl;
    __syncthreads();
    T off = T(0), tot = T(0);
#pragma unroll 4
    for (int k = 0; k < W; ++k) {
      const T p = sm[team * W + k];
      if (k < wit) off = OpSum::apply(off, p);
      tot = OpSum::apply(tot, p);
    }
    __syncthreads();
    *total = tot;
    return OpSum::apply(off, wexcl);
  }
  // read_from_master through a per-team shared slot.
  template <class T>
  __device__ __forceinline__ T read_from_master(T v, T* slot /*[teams]*/) const {
    if (slave == 0) slot[team] = v;
    __syncthreads();
    const T r = slot[team];
    __syncthreads();
    return r;
  }
};

template <int S> struct MultiShape {
  static constexpr int CTA = S < 256 ? 256 : S;  // threads per CTA
  static constexpr int TEAMS = CTA / S;          // teams (items) per CTA
  static constexpr int MINB = 1024 / CTA;        // CTAs per SM -> 64 registers/thread
};

}  // namespace cudanp
