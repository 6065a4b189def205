// bf16 / fp16 path: persistent, warp-specialised sm_100a kernel that walks the batching
// engine's work lists (Fig. 7, P294-312) with TMA-staged operands and tcgen05
// tensor-core MMA accumulating in TMEM.
//
// One CTA per SM (grid = min(Block_NUM, #SMs)), 16 warps:
//   warp 0      scheduler: starts with block = CTA index, then claims blocks (work lists)
//               with an atomic, software-pipelined one block ahead (the pair kernel claims
//               each block just in time, reading C-27); loads their tile
//               descriptors (one 32-byte record per tile, lanes in parallel) into a 32-entry
//               smem tile ring and prefetches the tiles' tensor maps; lookahead is bounded in
//               k-blocks so the GPU works on a short window of GEMMs at a time (L2 reuse of A/B).
//   warp 1      TMEM owner + MMA issuer: one thread issues tcgen05.mma (M = BY, N = BX,
//               K = 16; a 256 x 512 W2 pair tile issues two N = 256 MMAs per K step) into an
//               accumulator ring of 512 TMEM columns (up to 8 tiles in flight).
//   warps 2-3   C_old producers: TMA-load C_old chunks (BY x 64) per epilogue quarter into a
//               4-slot ring when beta != 0 (C is never read when beta == 0, reading C-16).
//   warps 4-7   A/B producers: stream each tile's k-blocks (A: BY x 64, B: 64 x BX; for an
//               implicit-GEMM convolution tile A comes from TMA im2col copies) with TMA
//               into a PAGED ring (18 pages of 8 KB; a k-block takes 2 pages for 64x32 ... 6
//               for 128x256, so small tiles keep up to 9 k-blocks in flight — the paper's ILP
//               concern for small K, P151/P259, as TMA depth).  One thread issues only ~1 TMA
//               box per 250 cycles, so four warps split every k-block's boxes.
//   warps 8-15  epilogue: warps 8+q and 12+q own TMEM lane quarter q and split each chunk's
//               columns; tcgen05.ld, C = alpha*acc + beta*C_old in fp32, RNE to bf16/fp16 in
//               the swizzled smem chunk, TMA store of the quarter's sub-box (completion
//               deferred one chunk); the accumulator is released after its last tcgen05.ld.
// The paper's "unified thread structure" (P181) becomes a runtime MMA instruction descriptor
// per tile, so one kernel serves every strategy of the table.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "plan_types.h"
#include "sm100.cuh"

namespace vb {
namespace tck {

constexpr int kThreads = 512;              // 16 warps: see the role table in the header comment
#ifndef VB_NPROD
#define VB_NPROD 4
#endif
constexpr int kProducers = VB_NPROD;       // A/B TMA issuing warps (one thread issues ~1 box / 250 cycles)
constexpr int kCProducers = 2;             // C_old TMA issuing warps
constexpr int kBK = 64;                    // bf16 elements per k-block = one 128-B swizzle row
constexpr int kPageBytes = 8192;
#ifndef VB_PAGES
#define VB_PAGES 18
#endif
#ifndef VB_CSLOTS
#define VB_CSLOTS 4
#endif
#ifndef VB_KBAHEAD
#define VB_KBAHEAD 8
#endif
#ifndef VB_KB_PREFETCH
#define VB_KB_PREFETCH 0   // experiment: L2 prefetch of each A/B box this many k-blocks ahead
#endif
#ifndef VB_PREFETCH_TAILS
#define VB_PREFETCH_TAILS 1   // prefetch the tail maps a tile uses, and (pair) the peer SM's maps
#endif
#ifndef VB_JIT_CLAIM
#define VB_JIT_CLAIM 1   // pair kernel: claim each block just in time (reading C-27)
#endif
#ifndef VB_EPI_FFMA2
#define VB_EPI_FFMA2 1   // epilogue alpha*acc + beta*C_old as paired fp32 FMUL2/FFMA2 (0: scalar)
#endif
#ifndef VB_A_NEXT_PREFETCH
#define VB_A_NEXT_PREFETCH 0   // experiment: L2 prefetch of the next k-block's A box at even k-blocks
#endif
#ifndef VB_C_NEXT_PREFETCH
#define VB_C_NEXT_PREFETCH 0   // experiment: L2 prefetch of the next C_old chunk at even chunks
#endif
#ifndef VB_A_PAIR_PREFETCH
#define VB_A_PAIR_PREFETCH 0   // experiment: L2 prefetch of the A box 2 k-blocks ahead at even k-blocks
#endif
// L2 evict-first hints on the C_old loads / C stores.  Measured off by default: with the load
// hint, C5 read 1.3x its compulsory DRAM bytes (a 500^3 batch: C_old fetched ~1.6x) and ran
// 6% slower; without it DRAM reads are within 1-2% of the compulsory bytes.
#ifndef VB_CLOAD_HINT
#define VB_CLOAD_HINT 0
#endif
#ifndef VB_CSTORE_HINT
#define VB_CSTORE_HINT 0
#endif
#ifndef VB_AB_HINT
#define VB_AB_HINT 0      // experiment: A/B loads marked L2 evict-last
#endif
#ifndef VB_NGRAN
#define VB_NGRAN 16
#endif
constexpr int kNGran = VB_NGRAN;          // MMA N granularity per CTA for edge tiles (power of 2)
#ifndef VB_PAGES_PAIR
#define VB_PAGES_PAIR VB_PAGES
#endif
#ifndef VB_CSLOTS_PAIR
#define VB_CSLOTS_PAIR VB_CSLOTS
#endif
// Shared-memory split between the A/B page ring and the C slots, per kernel (experiment switches
// VB_PAGES_PAIR / VB_CSLOTS_PAIR give the pair kernel its own split; by default both kernels use
// 18 pages + 4 C slots).
template <bool PAIR> struct Layout {
  static constexpr int kPages = PAIR ? VB_PAGES_PAIR : VB_PAGES;
  static constexpr int kCSlots = PAIR ? VB_CSLOTS_PAIR : VB_CSLOTS;
  // a layout at the 227 KB opt-in limit has no alignment slack: the kernel then checks that
  // dynamic shared memory starts 1024-byte aligned (SW128 atoms) and traps if not
  static constexpr int kSlack = (kPages * 8192 + kCSlots * 16384 + 4096 > 232448 - 1024) ? 0 : 1024;
};
constexpr int kSlots = 16;                 // k-blocks in flight (bounded by pages anyway)
constexpr int kCSlotsMax = VB_CSLOTS > VB_CSLOTS_PAIR ? VB_CSLOTS : VB_CSLOTS_PAIR;
static_assert(VB_CSLOTS >= 2 && VB_CSLOTS_PAIR >= 2,
              "the epilogue defers each store's completion by one chunk: one C slot deadlocks");
constexpr int kCSlotBytes = 128 * 128;     // BY rows x 128 B
constexpr int kRing = 32;                  // tile-descriptor ring entries
constexpr int kKbAhead = VB_KBAHEAD;       // scheduler lookahead budget in k-blocks (L2 locality)
constexpr int kTmemCols = 512;
constexpr int kAccUnit = 32;               // TMEM accumulator ring granularity (columns)
constexpr int kAccUnits = kTmemCols / kAccUnit;
constexpr int kAcc = 8;                    // accumulators in flight (ring entries)
#ifndef VB_ACC_SPLIT
#define VB_ACC_SPLIT 1   // 1: in the 1-SM kernel, 2: in both kernels, 0: off
#endif
// Accumulators of 8+ units as two ring entries (halves): the epilogue hands the first half back
// as soon as it is drained, so a following tile that fits there starts its MMAs early.  Measured
// (paired rounds): C5 0.99 (1-SM kernel, short-K tiles with 128-column neighbours), C4 1.015 when
// also used by the pair kernel (its W2 neighbours rarely fit in a half) -- so 1-SM only.
// Returns the units of the first half, 0 = not split (a half is whole 64-column epilogue chunks).
template <bool PAIR>
__device__ __forceinline__ int split_units(int units) {
  const bool on = PAIR ? VB_ACC_SPLIT == 2 : VB_ACC_SPLIT != 0;
  return (on && units >= 8 && (units & 3) == 0) ? units / 2 : 0;
}
constexpr int kEpiWarps = 8;               // two per TMEM lane quarter, splitting each chunk's columns
constexpr uint32_t kRingConsumers = kProducers + 1 + kCProducers + kEpiWarps;

struct TileInfo {          // one tile ring entry (48 bytes: three 16-byte DSMEM stores in a pair)
  TileDesc d;
  int32_t pad[4];
};
static_assert(sizeof(TileInfo) == 48, "TileInfo size");
// Opt-in timeline (build with -DVB_TIMELINE, measurement only): the first %globaltimer stamp
// of each event of CTA 0 into p.trace[i] (zeroed by the caller).  Events: 0 entry, 1 setup
// done, 2 first ring entry pushed, 3 first k-block armed by a producer, 4 MMA saw its first
// k-block, 5 first accumulator committed, 6 epilogue saw it, 7 epilogue done with it, 8 its
// stores complete, 9 teardown barrier passed, 10 exit.
#ifdef VB_TIMELINE_ALL
// Opt-in (measurement only): every CTA stores %globaltimer at entry and exit into
// p.trace[2 * blockIdx.x + {0, 1}] (the buffer holds 2 * gridDim.x entries).
__device__ __forceinline__ void vb_stamp_all(long long *buf, int i) {
  if (buf) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    buf[2 * blockIdx.x + i] = (long long)t;
  }
}
#endif
#ifdef VB_TIMELINE
__device__ __forceinline__ void vb_stamp(long long *buf, int i) {
  if (blockIdx.x == 0 && buf) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    atomicCAS(reinterpret_cast<unsigned long long *>(buf) + i, 0ull, t);
  }
}
#define VB_STAMP(i) vb_stamp(p.trace, i)
#else
#define VB_STAMP(i)
#endif

struct Shared {
  uint64_t full[kSlots], empty[kSlots];
  uint64_t tfull[kAcc], tempty[kAcc];
  uint64_t cfull[kCSlotsMax], cempty[kCSlotsMax];
  uint64_t rfull[kRing], rempty[kRing];
  int32_t slot_page[kSlots];
  int32_t slot_pages[kProducers][kSlots];   // per producer replica: pages charged per k-block
  int32_t acc_take[kAcc];       // MMA-private: TMEM units charged to each accumulator in flight
  uint32_t tmem_base;
  uint32_t prod_kb;             // k-blocks (>= 1 per tile) the A/B producer has finished issuing (atomics only)
  TileInfo ring[kRing];
};

template <bool PAIR>
constexpr size_t smem_bytes() {
  return (size_t)Layout<PAIR>::kSlack + (size_t)Layout<PAIR>::kPages * kPageBytes +
         (size_t)Layout<PAIR>::kCSlots * kCSlotBytes + ((sizeof(Shared) + 127) / 128) * 128;
}
static_assert(smem_bytes<true>() <= 232448 && smem_bytes<false>() <= 232448, "over the 227 KB opt-in limit");

// Opt-in cycle accounting (build with -DVB_TRACE): per-CTA cycles each role spends waiting
// on each barrier, accumulated into TcArgs::trace[kTraceSlots] (unused in product builds).
enum TraceSlot {
  T_SCHED_REMPTY, T_SCHED_BUDGET, T_PROD_RFULL, T_PROD_EMPTY, T_MMA_RFULL, T_MMA_TEMPTY, T_MMA_FULL,
  T_CPROD_RFULL, T_CPROD_CEMPTY, T_EPI_RFULL, T_EPI_TFULL, T_EPI_CFULL, T_EPI_STORE, T_EPI_TMEM, T_EPI_MATH,
  T_TOTAL, T_TILES, T_PROD_ISSUE, T_MMA_ISSUE, T_EPI_FENCEBAR, T_EPI_STISSUE, T_EPI_LOOP,
  T_EPI_TLOAD, T_EPI_REL, T_EPI_PROC, T_EPI_HEAD, kTraceSlots
};
#ifdef VB_TRACE
#define VB_T0() const long long _vbt0 = clock64()
#define VB_TADD(slot) tr[slot] += clock64() - _vbt0
#define VB_TWAIT(slot, stmt) \
  do {                       \
    VB_T0();                 \
    stmt;                    \
    VB_TADD(slot);           \
  } while (0)
#else
#define VB_T0()
#define VB_TADD(slot)
#define VB_TWAIT(slot, stmt) stmt
#endif

__device__ __forceinline__ int geo_BY(uint16_t g) { return (g & 0xFF) * 16; }
__device__ __forceinline__ int geo_BX(uint16_t g) { return (g >> 8) * 16; }

// MMA width of a tile: a tile at the right edge of its GEMM computes only the columns up to N,
// rounded up to kNGran per CTA (a pair tile splits them evenly: CTA r supplies B columns
// n0 + r * n/2 ..).  The columns past it are never stored, so tensor time on them is waste.
__device__ __forceinline__ int mma_cols(int BX, int N, int n0, bool pair) {
  const int g = pair ? 2 * kNGran : kNGran;
  const int cols = min(BX, N - n0);
  return min(BX, (cols + g - 1) & ~(g - 1));
}
// MMA N of half h of a tile whose MMA width is mc: a W2 pair tile (BX = 512) issues two MMAs
// per K step, half h covering the tile's columns [256h, 256h + width) into TMEM columns
// [256h, ..); every other tile has one half (mc <= 256).
__device__ __forceinline__ int half_cols(int mc, int h) { return h == 0 ? min(mc, 256) : max(0, mc - 256); }
// shared-memory bytes between the two halves' B panels of one CTA (128 columns x BK rows)
constexpr int kHalfBBytes = 128 * 64 * 2;
// TMEM columns (32-column units) an accumulator occupies: its MMA width rounded up to whole
// epilogue chunks (the epilogue reads every column of a live chunk), not BX, so tiles at the
// right edge of narrow GEMMs leave room for more accumulators in flight
__device__ __forceinline__ int acc_units(int BX, int N, int n0, bool pair) {
  const int cc = BX >= 64 ? 64 : BX;
  return ((mma_cols(BX, N, n0, pair) + cc - 1) / cc) * cc / kAccUnit;
}
// Swap-AB tile: the MMA's N = the tile's C rows below M, rounded up to 16 (<= BY)
__device__ __forceinline__ int swap_rows(const TileDesc &d) {
  return min(geo_BY(d.geo), (d.M - d.m0 + 15) & ~15);
}
// TMEM units (32 columns) of a tile's accumulator
__device__ __forceinline__ int tile_acc_units(const TileDesc &d, bool pair, bool swap_kernel) {
  if (swap_kernel && (d.flags & kFlagSwap)) return (swap_rows(d) + kAccUnit - 1) / kAccUnit;
  return acc_units(geo_BX(d.geo), d.N, d.n0, pair);
}
// C chunks of a tile that hold any column < N (the epilogue and C producer skip the rest)
__device__ __forceinline__ int live_chunks(const TcGeom &geo, int N, int n0) {
  const int cols = min(geo.BX, N - n0);
  return min(geo.c_chunks, (cols + geo.c_cols - 1) >> (__ffs(geo.c_cols) - 1));
}

// TMEM accumulator ring: tile t takes BX/32 contiguous 32-column units starting at `head`
// (never wrapping); the MMA warp and the epilogue run this same function over the same tile
// sequence, so the epilogue knows each accumulator's columns without any message.
struct AccRing {
  int head = 0;
  __device__ __forceinline__ int place(int units, int &take) {
    int start = head;
    take = units;
    if (start + units > kAccUnits) {
      // charge the skipped end of the ring too; a 512-column accumulator (W2) overlaps it, and
      // the charge is the union of the two regions (the whole ring)
      take += kAccUnits - start - max(0, units - start);
      start = 0;
    }
    head = start + units;
    if (head == kAccUnits) head = 0;
    return start;
  }
};

__device__ __forceinline__ void advance(int &idx, uint32_t &phase, int n) {
  if (++idx == n) {
    idx = 0;
    phase ^= 1u;
  }
}

// ------------------------------------------------------------------------- epilogue math
template <int AB_FMT>
__device__ __forceinline__ void unpack8(uint4 w, float (&f)[8]) {
  const uint32_t u[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    if constexpr (AB_FMT == 1) {
      // bf16 -> fp32 is exact and is the bf16 bits in the top half: one SHL / LOP3 each
      f[2 * i] = __uint_as_float(u[i] << 16);
      f[2 * i + 1] = __uint_as_float(u[i] & 0xFFFF0000u);
    } else {
      const float2 v = __half22float2(*reinterpret_cast<const __half2 *>(&u[i]));
      f[2 * i] = v.x;
      f[2 * i + 1] = v.y;
    }
  }
}

template <int AB_FMT>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  if constexpr (AB_FMT == 1) {
    __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
    return *reinterpret_cast<uint32_t *>(&h);
  } else {
    __half2 h = __floats2half2_rn(lo, hi);
    return *reinterpret_cast<uint32_t *>(&h);
  }
}

// One C element (bf16 / fp16 bits) <-> fp32; the store rounds to nearest even (C-17).
template <int AB_FMT>
__device__ __forceinline__ float c_to_float(uint16_t b) {
  if constexpr (AB_FMT == 1)
    return __bfloat162float(__ushort_as_bfloat16(b));
  else
    return __half2float(__ushort_as_half(b));
}
template <int AB_FMT>
__device__ __forceinline__ uint16_t float_to_c(float x) {
  if constexpr (AB_FMT == 1)
    return __bfloat16_as_ushort(__float2bfloat16_rn(x));
  else
    return __half_as_ushort(__float2half_rn(x));
}

// NU 16-byte units (8 outputs each) of this thread's row of one C chunk, starting at unit
// u0, in place in smem.  All C_old units are read first, then computed, then written, so the
// shared-memory accesses do not form one serial read-modify-write chain.
template <int AB_FMT, int NU>
__device__ __forceinline__ void epi_row(uint8_t *cb, int row, int c_swz, int u0, const uint32_t *acc, float alpha,
                                        float beta) {
  uint32_t off[NU];
#pragma unroll
  for (int u = 0; u < NU; ++u) off[u] = ptx::swz((uint32_t)(row * c_swz + (u0 + u) * 16), c_swz);
  uint4 w[NU];
  if (beta != 0.f) {
#pragma unroll
    for (int u = 0; u < NU; ++u) w[u] = *reinterpret_cast<const uint4 *>(cb + off[u]);
#pragma unroll
    for (int u = 0; u < NU; ++u) {
      float old[8], o[8];
      unpack8<AB_FMT>(w[u], old);
#if VB_EPI_FFMA2
      // paired fp32 ops (FMUL2 / FFMA2): the same two roundings per element as the scalar form
#pragma unroll
      for (int e = 0; e < 8; e += 2) {
        const float2 bo = __fmul2_rn(make_float2(beta, beta), make_float2(old[e], old[e + 1]));
        const float2 r = __ffma2_rn(make_float2(alpha, alpha),
                                    make_float2(__uint_as_float(acc[u * 8 + e]), __uint_as_float(acc[u * 8 + e + 1])), bo);
        o[e] = r.x;
        o[e + 1] = r.y;
      }
#else
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = fmaf(alpha, __uint_as_float(acc[u * 8 + e]), beta * old[e]);
#endif
      w[u].x = pack2<AB_FMT>(o[0], o[1]);
      w[u].y = pack2<AB_FMT>(o[2], o[3]);
      w[u].z = pack2<AB_FMT>(o[4], o[5]);
      w[u].w = pack2<AB_FMT>(o[6], o[7]);
    }
  } else {
#pragma unroll
    for (int u = 0; u < NU; ++u) {
      w[u].x = pack2<AB_FMT>(alpha * __uint_as_float(acc[u * 8 + 0]), alpha * __uint_as_float(acc[u * 8 + 1]));
      w[u].y = pack2<AB_FMT>(alpha * __uint_as_float(acc[u * 8 + 2]), alpha * __uint_as_float(acc[u * 8 + 3]));
      w[u].z = pack2<AB_FMT>(alpha * __uint_as_float(acc[u * 8 + 4]), alpha * __uint_as_float(acc[u * 8 + 5]));
      w[u].w = pack2<AB_FMT>(alpha * __uint_as_float(acc[u * 8 + 6]), alpha * __uint_as_float(acc[u * 8 + 7]));
    }
  }
#pragma unroll
  for (int u = 0; u < NU; ++u) *reinterpret_cast<uint4 *>(cb + off[u]) = w[u];
}

// --------------------------------------------------------------------------------- kernel
// SWAP = the 1-SM variant that also runs swap-AB tiles (launched only for plans that have them,
// so the other plans do not carry its epilogue path).
// PAIR = the 2-SM variant (cluster of 2 CTAs, cta_group::2): every tile is a 256-row pair tile,
// CTA r owns rows r*128.. of it and half of B; CTA 0 (the leader) schedules, issues the MMAs and
// owns the barriers both CTAs' TMA loads and epilogues report to.
template <int AB_FMT, bool PAIR, bool SWAP = false>
__global__ void __launch_bounds__(kThreads, 1) vb_tc_kernel(const __grid_constant__ TcArgs p) {
  constexpr int kPages = Layout<PAIR>::kPages, kCSlots = Layout<PAIR>::kCSlots;
  extern __shared__ uint8_t smem_raw[];
  if (Layout<PAIR>::kSlack == 0 && (ptx::smem_u32(smem_raw) & 1023u) != 0u) __trap();
  // 1024-byte aligned (SW128 atoms); offsetting smem_raw itself keeps the shared address space
  // visible to the compiler, so C-slot and barrier accesses compile to LDS/STS, not generic LD/ST.
  uint8_t *smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  if (threadIdx.x == 0) VB_STAMP(0);
#ifdef VB_TIMELINE_ALL
  if (threadIdx.x == 0) vb_stamp_all(p.trace, 0);
#endif
  uint8_t *pages = smem;
  uint8_t *cbuf = smem + (size_t)kPages * kPageBytes;
  Shared *sh = reinterpret_cast<Shared *>(cbuf + (size_t)kCSlots * kCSlotBytes);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const uint32_t rank = PAIR ? ptx::cluster_ctarank() : 0u;
  const bool leader = rank == 0;
  // in a pair, consumers of the peer CTA release ring entries / accumulators on the leader
  // Every consumer releases a ring entry on its own CTA's barrier (a CTA-scope arrive).  In a
  // pair, one forwarding thread of the peer CTA waits for the peer's local releases and passes
  // each on to the leader with a single cluster-scope arrive: the producer, C-producer and
  // epilogue warps of the peer never issue a release.cluster arrive themselves, which first
  // waits for the thread's outstanding memory operations to be performed at cluster scope
  // (measured: the per-warp remote arrives cost C4 ~4 %).  Accumulator releases need no memory
  // ordering (the TMEM reads are complete, nothing is published): the peer's epilogue warps
  // arrive on the leader's barrier with relaxed remote arrives.
  auto ring_release = [&](int e) { ptx::mbar_arrive(&sh->rempty[e]); };
  // the leader's ring entries are written by its own scheduler (CTA scope); the peer's by the
  // leader's scheduler through DSMEM (cluster scope)
  // warm this SM's TMA descriptor cache for a tile's maps well before its producers use them
  // (the row-tail and K-tail maps too, when the tile uses them: a tile's first k-block or its
  // last one would otherwise wait for a descriptor fetch)
  auto prefetch_tile_maps = [&](const TileDesc &d) {
    const uint8_t *maps = reinterpret_cast<const uint8_t *>(p.tmaps) + (size_t)d.gemm * (kMapsPerGemm * 128);
    if (d.kblocks > 0) {
      ptx::prefetch_tmap(maps + MAP_A * 128);
      ptx::prefetch_tmap(maps + MAP_B * 128);
#if VB_PREFETCH_TAILS
      const int BYc = geo_BY(d.geo) / (PAIR ? 2 : 1);
      if (d.M % BYc != 0 && d.m0 + geo_BY(d.geo) > d.M) ptx::prefetch_tmap(maps + MAP_A_TAIL * 128);
      if (!(d.flags & kFlagConv) && ((d.flags >> 8) & 7) != 0) ptx::prefetch_tmap(maps + MAP_B_TAIL * 128);
#endif
    }
    ptx::prefetch_tmap(maps + MAP_C * 128);
    if (d.N >= 8) ptx::prefetch_tmap(maps + MAP_C_ST * 128);
  };
  auto ring_wait = [&](int e, uint32_t ph) {
    if (PAIR && !leader)
      ptx::mbar_wait_cluster(&sh->rfull[e], ph);
    else
      ptx::mbar_wait(&sh->rfull[e], ph);
  };

  if (threadIdx.x == 0) {
    for (int i = 0; i < kSlots; ++i) {
      ptx::mbar_init(&sh->full[i], 1);
      ptx::mbar_init(&sh->empty[i], 1);
    }
    for (int i = 0; i < kAcc; ++i) {
      ptx::mbar_init(&sh->tfull[i], 1);
      ptx::mbar_init(&sh->tempty[i], PAIR ? 2 * kEpiWarps : kEpiWarps);
    }
    for (int i = 0; i < kCSlots; ++i) {
      ptx::mbar_init(&sh->cfull[i], kCProducers);
      ptx::mbar_init(&sh->cempty[i], 4);   // one arrival per lane quarter (its storing warp)
    }
    for (int i = 0; i < kRing; ++i) {
      ptx::mbar_init(&sh->rfull[i], 1);
      // leader: its own consumers + the peer's forwarder; peer: its consumers (it has no MMA thread)
      ptx::mbar_init(&sh->rempty[i], PAIR ? (leader ? kRingConsumers + 1 : kRingConsumers - 1) : kRingConsumers);
    }
    sh->prod_kb = 0u;
    ptx::fence_mbar_init();
  }
  // pair: both CTAs' shared-memory initialisation is complete (cluster-wide) before the
  // cta_group::2 allocation, which writes the TMEM address into shared memory asynchronously
  // (compute-sanitizer racecheck reports the allocation against the initialisation otherwise)
  if (PAIR) ptx::cluster_sync();
  if (warp == 1) {
    if (PAIR)
      ptx::tmem_alloc_pair(&sh->tmem_base, kTmemCols);
    else
      ptx::tmem_alloc(&sh->tmem_base, kTmemCols);
  }
  ptx::tc_fence_before();
  if (PAIR)
    ptx::cluster_sync();   // both CTAs' barriers initialised before any remote arrive
  else
    __syncthreads();
  ptx::tc_fence_after();
#ifndef VB_NO_PDL
  // programmatic dependent launch: the setup above overlapped the bind-time prep kernel; the
  // tensor maps it patches and the work-list counters it resets are used only after this wait
  asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
  const uint32_t tmem_base = sh->tmem_base;
  if (threadIdx.x == 0) VB_STAMP(1);
  const uint8_t *tmaps = reinterpret_cast<const uint8_t *>(p.tmaps);
#ifdef VB_TRACE
  long long tr[kTraceSlots];
  for (int i = 0; i < kTraceSlots; ++i) tr[i] = 0;
  const long long t_start = clock64();
#endif

  if (warp == 0 && leader) {
    // ================================================================ scheduler (whole warp)
    // Tile t of this CTA goes to ring entry t % kRing with phase (t / kRing) & 1.
    // The lookahead is bounded in k-blocks (kKbAhead) rather than tiles, so CTAs working on
    // long-K tiles do not hoard blocks: the blocks in progress across the GPU stay a short
    // window of consecutive GEMMs and their A/B re-reads hit in L2.
    uint32_t t = 0, pushed_kb = 0;
    // the first block of every CTA (cluster) is static -- block = CTA (cluster) index -- so the
    // first tile's descriptor read does not wait for an atomic round trip; later blocks are
    // claimed from the counter, offset by the number of CTAs (clusters)
    const int n_static = (int)gridDim.x / (PAIR ? 2 : 1);
    // Software-pipelined by one block: while the tiles of block b are read and pushed, the
    // CSR range of the next block (claimed one ahead) is already in flight and the block after
    // it is being claimed, so each block costs one dependent global round trip, not three.
    //
    // The pair kernel (kJitClaim) instead claims each block just in time: after pushing a block
    // it waits for the lookahead budget and only then claims the next one (reading C-27).  Its
    // blocks hold long tiles (tens of microseconds); a block claimed two ahead starts up to two
    // block durations after its claim, so the tiles of one GEMM -- claimed back to back by
    // different pairs -- would start that far apart and re-read their shared A / B panels from
    // DRAM.  The claim's two round trips (counter, block range) hide behind the kKbAhead k-blocks
    // already pushed.
    constexpr bool kJitClaim = (PAIR && VB_JIT_CLAIM) || VB_JIT_CLAIM == 2;
    int b = (int)blockIdx.x / (PAIR ? 2 : 1);
    int lim = (b < p.n_blocks && lane < 2) ? p.block_ptr[b + lane] : 0;
    int nb = 0;
    if (!kJitClaim && lane == 0) nb = n_static + atomicAdd(p.counter, 1);
    nb = __shfl_sync(0xffffffffu, nb, 0);
    for (;;) {
      if (b >= p.n_blocks) break;
      int nb2 = nb;
      if (!kJitClaim && lane == 0) {
        VB_TWAIT(T_SCHED_BUDGET, while ((int)(pushed_kb - atomicAdd(&sh->prod_kb, 0u)) > kKbAhead) __nanosleep(128));
        if (nb < p.n_blocks) nb2 = n_static + atomicAdd(p.counter, 1);   // claim two ahead
      }
      int lim_next = (!kJitClaim && nb < p.n_blocks && lane < 2) ? p.block_ptr[nb + lane] : 0;
      const int s0 = __shfl_sync(0xffffffffu, lim, 0), s1 = __shfl_sync(0xffffffffu, lim, 1);
      for (int base = s0; base < s1; base += 32) {
        const int n = min(32, s1 - base);
        int kb = 0;
        if (lane < n) {
          const TileDesc d = p.tiles[base + lane];
          kb = max(d.kblocks, 1);
          // warm the TMA descriptor cache for the tile's maps well before the producers use them
          prefetch_tile_maps(d);
          const uint32_t tt = t + lane;
          const int e = (int)(tt % kRing);
          VB_TWAIT(T_SCHED_REMPTY, ptx::mbar_wait(&sh->rempty[e], ((tt / kRing) & 1u) ^ 1u));
          TileInfo &ti = sh->ring[e];
          ti.d = d;   // alpha / beta are read by their users (C producers, epilogue) off this chain
          if (PAIR) {                                 // mirror the entry into the peer's ring
            const uint32_t ra = ptx::mapa(&ti, 1);
            const uint4 *src = reinterpret_cast<const uint4 *>(&ti);
            ptx::st_cluster_v4(ra, src[0]);
            ptx::st_cluster_v4(ra + 16, src[1]);
            ptx::st_cluster_v4(ra + 32, src[2]);
            ptx::mbar_arrive_remote(ptx::mapa(&sh->rfull[e], 1));
          }
          ptx::mbar_arrive(&sh->rfull[e]);
          VB_STAMP(2);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) kb += __shfl_xor_sync(0xffffffffu, kb, o);
        pushed_kb += (uint32_t)kb;
        t += (uint32_t)n;
      }
      if (kJitClaim) {
        if (lane == 0) {
          VB_TWAIT(T_SCHED_BUDGET, while ((int)(pushed_kb - atomicAdd(&sh->prod_kb, 0u)) > kKbAhead) __nanosleep(128));
          nb = n_static + atomicAdd(p.counter, 1);
        }
        nb = __shfl_sync(0xffffffffu, nb, 0);
        lim_next = (nb < p.n_blocks && lane < 2) ? p.block_ptr[nb + lane] : 0;
        b = nb;
        lim = lim_next;
      } else {
        b = nb;
        lim = lim_next;
        nb = __shfl_sync(0xffffffffu, nb2, 0);
      }
    }
    if (lane == 0) {                                        // end marker
      const int e = (int)(t % kRing);
      ptx::mbar_wait(&sh->rempty[e], ((t / kRing) & 1u) ^ 1u);
      sh->ring[e].d.gemm = -1;
      if (PAIR) {
        asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(ptx::mapa(&sh->ring[e].d.gemm, 1)), "r"(-1) : "memory");
        ptx::mbar_arrive_remote(ptx::mapa(&sh->rfull[e], 1));
      }
      ptx::mbar_arrive(&sh->rfull[e]);
    }
  } else if (warp == 0) {
    // ================================================================ peer: ring-release forwarder
    // the peer CTA of a pair has no scheduler (the leader mirrors every ring entry into it); its
    // warp 0 forwards each entry's release, once all the peer's consumers have made it
    if (PAIR && lane == 0) {
      for (uint32_t t = 0;; ++t) {
        const int e = (int)(t % kRing);
        const uint32_t ph = (t / kRing) & 1u;
        ring_wait(e, ph);
        const bool end = sh->ring[e].d.gemm < 0;
#if VB_PREFETCH_TAILS
        if (!end) prefetch_tile_maps(sh->ring[e].d);   // the peer SM's own descriptor cache
#endif
        ptx::mbar_wait(&sh->rempty[e], ph);
        ptx::mbar_arrive_remote(ptx::mapa(&sh->rempty[e], 0));
        if (end) break;
      }
    }
  } else if (warp >= 4 && warp < 8) {
    // ================================================================ A/B TMA producers
    // kProducers warps run the same deterministic page allocator over the same tile sequence
    // (so they agree on every k-block's pages without talking) and split each k-block's TMA
    // boxes round-robin: one thread can issue only ~1 box per 250 cycles.  Producer 0 alone
    // arms the full barrier (arrive + expect_tx of the k-block's total bytes), publishes the
    // k-block's page, and reports progress to the scheduler.
    const int pid = warp - 4;
    const uint64_t ab_policy = ptx::policy_evict_last();
    (void)ab_policy;
    if (lane == 0 && pid < kProducers) {
      int re = 0, slot = 0, head = 0, oldest = 0, inflight = 0, free_pages = kPages;
      uint32_t rph = 0, sph = 0, ophase = 0, kbg = 0;
      int32_t *slot_pages = sh->slot_pages[pid];
      for (;;) {
        VB_TWAIT(T_PROD_RFULL, ring_wait(re, rph));
        const TileInfo ti = sh->ring[re];
        ring_release(re);
        advance(re, rph, kRing);
        if (ti.d.gemm < 0) break;
        if (ti.d.kblocks == 0) {
          if (pid == 0 && leader) atomicAdd(&sh->prod_kb, 1u);   // flow control for the scheduler
          continue;
        }
        // per-CTA geometry: a pair tile gives each CTA 128 rows of A and BX/2 columns of B
        const int BY = geo_BY(ti.d.geo) / (PAIR ? 2 : 1), BX = geo_BX(ti.d.geo);
        const int BXc = PAIR ? min(BX, 256) / 2 : BX;   // B columns of one MMA half in this CTA
        const TcGeom geo = tc_geom(BY, BXc);
        // MMA halves (two for a W2 tile): half h's B columns per CTA (a pair splits each evenly)
        const int mc = mma_cols(BX, ti.d.N, ti.d.n0, PAIR);
        const int Nh0 = half_cols(mc, 0) / (PAIR ? 2 : 1), Nh1 = half_cols(mc, 1) / (PAIR ? 2 : 1);
        const uint8_t *maps = tmaps + (size_t)ti.d.gemm * (kMapsPerGemm * 128);
        // out-of-bounds box rows cost L2 bandwidth even though TMA zero-fills them: the last
        // row-tile uses the row-tail map, the last k-block the K-tail map, and B boxes that lie
        // entirely past N are not loaded (their MMA columns are discarded by the epilogue)
        // rows / B boxes this CTA loads, and (pair) what the peer loads, for the byte count
        auto a_box_rows_of = [&](int r) {
          const int rows = min(BY, ti.d.M - (ti.d.m0 + r * BY));
          return rows <= 0 ? 0 : (rows < BY ? (rows + 7) / 8 * 8 : BY);
        };
        auto b_boxes_half = [&](int r, int h) {
          const int nh = h ? Nh1 : Nh0;
          const int cols = min(nh, ti.d.N - (ti.d.n0 + h * 256 + r * nh));
          const int bw = geo.b_swz / 2;                  // a power of two: shift, not divide
          return cols <= 0 ? 0 : min(geo.b_boxes, (cols + bw - 1) >> (__ffs(bw) - 1));
        };
        auto b_boxes_of = [&](int r) { return b_boxes_half(r, 0) + (Nh1 ? b_boxes_half(r, 1) : 0); };
        const int row0 = ti.d.m0 + (int)rank * BY;
        const int a_box_rows = a_box_rows_of((int)rank);
        const bool a_tail = a_box_rows != BY;
        const uint8_t *mapA = maps + (a_tail ? MAP_A_TAIL : MAP_A) * 128;
        const int b_boxes0 = b_boxes_half((int)rank, 0);
        const int b_boxes = b_boxes_of((int)rank);
        const int ksteps_last = (ti.d.flags >> 8) & 7;
        // implicit GEMM (vb_plan_conv): the window origin of this CTA's first output pixel
        const bool conv = (ti.d.flags & kFlagConv) != 0;
        ConvParam cv{};
        int img = 0, oy = 0, ox = 0, ctap = 0, ccb = 0;
        if (conv) {
          cv = p.conv[ti.d.gemm];
          const int hw = cv.Hout * cv.Wout;
          img = row0 / hw;
          const int rem = row0 - img * hw;
          oy = rem / cv.Wout;
          ox = rem - oy * cv.Wout;
        }
        const int a_pages = (BY * kBK * 2 + kPageBytes - 1) / kPageBytes;   // swap-AB tiles: 16-64 rows, 1 page
        const int b_span = Nh1 ? kHalfBBytes + Nh1 * kBK * 2 : Nh0 * kBK * 2;   // B panel bytes of this CTA
        const int need = a_pages + (b_span + kPageBytes - 1) / kPageBytes;
        // per-tile constants of the k-loop (the loop body is on the page-release -> TMA-issue
        // latency chain): transaction bytes of the A rows and the B box count of both CTAs, and
        // the first column of each MMA half's B boxes in this CTA
        const uint32_t a_tx = (uint32_t)((a_box_rows_of(0) + (PAIR ? a_box_rows_of(1) : 0)) * kBK * 2);
        const uint32_t b_box_tx = (uint32_t)((b_boxes_of(0) + (PAIR ? b_boxes_of(1) : 0)) * geo.b_swz);
        const int bcol0 = ti.d.n0 + (int)rank * Nh0, bcol1 = ti.d.n0 + 256 + (int)rank * Nh1;
        const int bstep = geo.b_swz / 2;
        for (int kb = 0; kb < ti.d.kblocks; ++kb, ++kbg) {
          int start = head, take = need;
          if (start + need > kPages) {          // never wrap a k-block around the ring end
            take += kPages - start;
            start = 0;
          }
          {
            VB_T0();
            while (free_pages < take || inflight == kSlots) {
              // reclaim the oldest k-block in flight once the MMA has consumed it
              ptx::mbar_wait(&sh->empty[oldest], ophase);
              free_pages += slot_pages[oldest];
              --inflight;
              advance(oldest, ophase, kSlots);
            }
            VB_TADD(T_PROD_EMPTY);
          }
          slot_pages[slot] = take;
          free_pages -= take;
          ++inflight;
          head = start + need;
          if (head == kPages) head = 0;
          const bool k_tail = !conv && (kb == ti.d.kblocks - 1) && ksteps_last != 0;   // conv: bits 8-10 mean per-tap steps
          const int b_rows = k_tail ? ksteps_last * 16 : kBK;
          const uint8_t *mapB = maps + (k_tail ? MAP_B_TAIL : MAP_B) * 128;
          uint8_t *sa = pages + (size_t)start * kPageBytes;
          uint8_t *sb = sa + (size_t)a_pages * kPageBytes;
          VB_T0();
          if (pid == 0) {
            sh->slot_page[slot] = start;
            if (leader) {                     // the leader's barrier counts both CTAs' bytes
              ptx::mbar_arrive_expect_tx(&sh->full[slot], a_tx + b_box_tx * (uint32_t)b_rows);
              VB_STAMP(3);
            }
          }
          // box 0 = A, boxes 1..b_boxes = B; box i goes to producer (i + kbg) % kProducers
          if (ptx::elect_lane0())
          for (int i = (int)(((uint32_t)pid - kbg) % (uint32_t)kProducers); i <= b_boxes; i += kProducers) {
            if (i == 0 && a_box_rows == 0) continue;
            // B box i - 1: box j of half h (half 1 at kHalfBBytes, columns 256 on)
            const int h = i - 1 >= b_boxes0 ? 1 : 0, j = i - 1 - h * b_boxes0;
            uint8_t *dst = i == 0 ? sa : sb + h * kHalfBBytes + j * kBK * geo.b_swz;
            const uint8_t *map = i == 0 ? mapA : mapB;
            if (conv) {   // k-block kb = (tap ctap, channel block ccb)
              if (i == 0) {
                const int kh = ctap / cv.KW, kw = ctap - kh * cv.KW;
                ptx::tma_load_im2col_4d(dst, map, &sh->full[slot], ccb * kBK, ox - cv.pad, oy - cv.pad, img,
                                        (uint16_t)kw, (uint16_t)kh);
              } else {
                ptx::tma_load_2d(dst, map, &sh->full[slot], ti.d.n0 + (int)rank * Nh0 + j * (geo.b_swz / 2),
                                 ctap * cv.Cin + ccb * kBK);
              }
              continue;
            }
            const int c0 = i == 0 ? kb * kBK : (h ? bcol1 : bcol0) + j * bstep;
            const int c1 = i == 0 ? row0 : kb * kBK;
            if (PAIR)
              ptx::tma_load_2d_pair(dst, map, &sh->full[slot], c0, c1);
            else
#if VB_AB_HINT
              ptx::tma_load_2d_hint(dst, map, &sh->full[slot], c0, c1, ab_policy);
#else
              ptx::tma_load_2d(dst, map, &sh->full[slot], c0, c1);
#endif
#if VB_A_PAIR_PREFETCH
            // even k-blocks: L2-prefetch the A box two k-blocks ahead, so that with the 256-byte L2
            // promotion DRAM sees 512 contiguous bytes of each A row requested together
            if (i == 0 && (kb & 1) == 0 && kb + 2 < ti.d.kblocks) ptx::tma_prefetch_2d(mapA, (kb + 2) * kBK, row0);
#endif
#if VB_A_NEXT_PREFETCH
            // even k-blocks: L2-prefetch the next k-block's A box right behind this one, so DRAM
            // sees 256 contiguous bytes of each A row requested together (a 128-byte box alone
            // streams at ~4.9 TB/s, two adjacent ones at ~7.3 TB/s: profiles/tma_locality_r01.txt)
            if (i == 0 && (kb & 1) == 0 && kb + 1 < ti.d.kblocks) ptx::tma_prefetch_2d(mapA, (kb + 1) * kBK, row0);
#endif
#if VB_KB_PREFETCH > 0
            // start the DRAM fetch of the same box VB_KB_PREFETCH k-blocks ahead into L2
            if (kb + VB_KB_PREFETCH < ti.d.kblocks) {
              const uint8_t *pmap = i == 0 ? mapA : maps + MAP_B * 128;
              if (i == 0)
                ptx::tma_prefetch_2d(pmap, (kb + VB_KB_PREFETCH) * kBK, row0);
              else
                ptx::tma_prefetch_2d(pmap, c0, (kb + VB_KB_PREFETCH) * kBK);
            }
#endif
          }
          VB_TADD(T_PROD_ISSUE);
          if (conv && ++ccb == cv.ncb) {
            ccb = 0;
            ++ctap;
          }
          advance(slot, sph, kSlots);
          if (pid == 0 && leader) atomicAdd(&sh->prod_kb, 1u);   // flow control for the scheduler
        }
      }
    }
  } else if (warp == 1) {
    // ================================================================ MMA issuer (+ TMEM owner)
    if (lane == 0 && leader) {
      int re = 0, slot = 0, oldest = 0, free_units = kAccUnits, inflight = 0;
      uint32_t rph = 0, sph = 0, t = 0, ophase = 0;
      int32_t *acc_take = sh->acc_take;
      AccRing ring;
      for (;;) {
        VB_TWAIT(T_MMA_RFULL, ring_wait(re, rph));
        const TileInfo ti = sh->ring[re];
        ring_release(re);
        advance(re, rph, kRing);
        if (ti.d.gemm < 0) break;
        const int BY = geo_BY(ti.d.geo), BX = geo_BX(ti.d.geo);   // MMA shape (pair: M = 256)
        const TcGeom geo = tc_geom(PAIR ? BY / 2 : BY, PAIR ? min(BX, 256) / 2 : BX);   // this CTA's B half
        // VB_ACC_SPLIT: an accumulator of 8+ units is two ring entries (halves); the epilogue hands
        // the first half back once drained, so a following tile that fits there starts early.
        const int units = tile_acc_units(ti.d, PAIR, SWAP);
        const int hu = split_units<PAIR>(units);
        const int nent = hu ? 2 : 1;
        const int e = (int)(t % kAcc), e1 = (int)((t + 1) % kAcc);
        t += (uint32_t)nent;
#ifdef VB_TRACE
        tr[T_TILES] += 1;
#endif
        int take;
        const int start = ring.place(units, take);
        {
          VB_T0();
          while (free_units < take || inflight + nent > kAcc) {   // reclaim drained accumulators (FIFO)
            ptx::mbar_wait(&sh->tempty[oldest], ophase);
            free_units += acc_take[oldest];
            --inflight;
            advance(oldest, ophase, kAcc);
          }
          VB_TADD(T_MMA_TEMPTY);
        }
        free_units -= take;
        if (nent == 2) {   // entry e: the skipped ring end (if any) + the first half; e1: the rest
          acc_take[e] = take - (units - hu);
          acc_take[e1] = units - hu;
        } else {
          acc_take[e] = take;
        }
        inflight += nent;
        ptx::tc_fence_after();
        const uint32_t d_tmem = tmem_base + (uint32_t)(start * kAccUnit);
        // swap-AB: A operand = the B panel (MN-major, M = BX = 128), B operand = the A rows
        // (K-major, N = the rows below M rounded to 16); the accumulator holds C^T
        const bool swap = SWAP && (ti.d.flags & kFlagSwap) != 0;
        const int mc = mma_cols(BX, ti.d.N, ti.d.n0, PAIR);
        const uint32_t idesc = swap ? ptx::idesc_f16_swap((uint32_t)AB_FMT, BX, swap_rows(ti.d))
                                    : ptx::idesc_f16((uint32_t)AB_FMT, BY, half_cols(mc, 0));
        // W2 pair tile: the second MMA half (columns 256.., B panel at kHalfBBytes, TMEM +256)
        const int mc1 = PAIR ? half_cols(mc, 1) : 0;
        const uint32_t idesc1 = mc1 ? ptx::idesc_f16((uint32_t)AB_FMT, BY, mc1) : 0u;
        const uint32_t blayout = ptx::swizzle_layout_code(geo.b_swz);
        // B follows A's pages (whole pages: a swap-AB tile's 16-64 A rows take one)
        const uint32_t a_bytes = (uint32_t)(((PAIR ? BY / 2 : BY) * kBK * 2 + kPageBytes - 1) / kPageBytes * kPageBytes);
        // descriptors of K step 0; step kk adds 32 B (A) / 16 rows * b_swz (B) to the start
        // address field (bits 0-13, address >> 4)
        const uint64_t adesc0 = ptx::smem_desc(0, 16, 1024, 2);
        const uint64_t bdesc0 = ptx::smem_desc(0, kBK * geo.b_swz, 8 * geo.b_swz, blayout);
        const uint32_t b_step = (uint32_t)geo.b_swz;    // (16 * b_swz) >> 4
        // implicit GEMM: the last channel block of every tap holds Cin % 64 channels; the K=16
        // steps past them would multiply zero-filled A columns and are skipped
        const bool conv = (ti.d.flags & kFlagConv) != 0;
        const int ncb = conv ? p.conv[ti.d.gemm].ncb : 0;
        int cb = 0;
        for (int kb = 0; kb < ti.d.kblocks; ++kb) {
          VB_TWAIT(T_MMA_FULL, ptx::mbar_wait(&sh->full[slot], sph));
          VB_STAMP(4);
          ptx::tc_fence_after();
          VB_T0();
          const uint32_t sa = ptx::smem_u32(pages + (size_t)sh->slot_page[slot] * kPageBytes);
          const uint32_t sb = sa + a_bytes;
          const int ksl = (ti.d.flags >> 8) & 7;
          const int ksteps = conv ? ((cb == ncb - 1 && ksl) ? ksl : kBK / 16)
                                  : ((kb == ti.d.kblocks - 1 && ksl) ? ksl : kBK / 16);
          if (conv && ++cb == ncb) cb = 0;
          const uint64_t adesc = adesc0 | (uint64_t)(sa >> 4);
          const uint64_t bdesc = bdesc0 | (uint64_t)(sb >> 4);
          if (ptx::elect_lane0()) {
#pragma unroll
            for (int kk = 0; kk < kBK / 16; ++kk) {
              if (kk >= ksteps) break;          // K tail: the B rows past the last step are not loaded
#ifndef VB_EXP_NOMMA
              if (PAIR) {
                ptx::mma_f16_ss_pair(d_tmem, adesc + 2u * kk, bdesc + b_step * kk, idesc, (kb | kk) != 0 ? 1u : 0u);
                if (mc1)
                  ptx::mma_f16_ss_pair(d_tmem + 256u, adesc + 2u * kk, bdesc + (uint32_t)(kHalfBBytes >> 4) + b_step * kk,
                                       idesc1, (kb | kk) != 0 ? 1u : 0u);
              } else if (SWAP && swap)
                ptx::mma_f16_ss(d_tmem, bdesc + b_step * kk, adesc + 2u * kk, idesc, (kb | kk) != 0 ? 1u : 0u);
              else
                ptx::mma_f16_ss(d_tmem, adesc + 2u * kk, bdesc + b_step * kk, idesc, (kb | kk) != 0 ? 1u : 0u);
#else
              (void)adesc; (void)bdesc; (void)idesc; (void)d_tmem;
#endif
            }
            if (PAIR)
              ptx::mma_commit_pair(&sh->empty[slot]);   // frees the k-block's pages in both CTAs
            else
              ptx::mma_commit(&sh->empty[slot]);      // frees the k-block's pages when the MMAs retire
          }
          VB_TADD(T_MMA_ISSUE);
          advance(slot, sph, kSlots);
        }
        if (ptx::elect_lane0()) {
          if (PAIR) {
            ptx::mma_commit_pair(&sh->tfull[e]);
            if (nent == 2) ptx::mma_commit_pair(&sh->tfull[e1]);
          } else {
            ptx::mma_commit(&sh->tfull[e]);         // accumulator ready for the epilogue
            if (nent == 2) ptx::mma_commit(&sh->tfull[e1]);
          }
          VB_STAMP(5);
        }
      }
    }
  } else if (warp == 2 || warp == 3) {
    // ================================================================ C_old producers
    // warp 2 loads the sub-boxes of lane quarters 0-1, warp 3 those of quarters 2-3
    const int cid = warp - 2;
    if (lane == 0) {
      int re = 0, cs = 0;
      uint32_t rph = 0, cph = 0;
      const uint64_t c_policy = ptx::policy_evict_first();
      (void)c_policy;
      for (;;) {
        VB_TWAIT(T_CPROD_RFULL, ring_wait(re, rph));
        const TileInfo ti = sh->ring[re];
        ring_release(re);
        advance(re, rph, kRing);
        if (ti.d.gemm < 0) break;
        if (SWAP && (ti.d.flags & kFlagSwap)) continue;  // swap-AB tiles read C_old directly
        const int BY = geo_BY(ti.d.geo) / (PAIR ? 2 : 1), BX = geo_BX(ti.d.geo);
        const TcGeom geo = tc_geom(BY, BX);
        const int row0 = ti.d.m0 + (int)rank * BY;
        const uint8_t *mapC = tmaps + (size_t)ti.d.gemm * (kMapsPerGemm * 128) + MAP_C * 128;
        const bool load = p.beta[ti.d.gemm] != 0.f;
        const int nch = live_chunks(geo, ti.d.N, ti.d.n0);
        for (int ch = 0; ch < nch; ++ch) {
          VB_TWAIT(T_CPROD_CEMPTY, ptx::mbar_wait(&sh->cempty[cs], cph ^ 1u));
          if (load && ptx::elect_lane0()) {
            // the C map's box is one epilogue quarter's sub-box (BY/4 rows); skip rows >= M
            const int rows_w = BY / 4;
            int nsub = 0;
            for (int w = 2 * cid; w < 2 * cid + 2; ++w) nsub += (row0 + w * rows_w < ti.d.M) ? 1 : 0;
            ptx::mbar_arrive_expect_tx(&sh->cfull[cs], (uint32_t)(nsub * rows_w * geo.c_cols * 2));
            for (int w = 2 * cid; w < 2 * cid + nsub; ++w)
#if VB_CLOAD_HINT
              ptx::tma_load_2d_hint(cbuf + (size_t)cs * kCSlotBytes + w * rows_w * geo.c_swz, mapC, &sh->cfull[cs],
                                    ti.d.n0 + ch * geo.c_cols, row0 + w * rows_w, c_policy);
#else
              ptx::tma_load_2d(cbuf + (size_t)cs * kCSlotBytes + w * rows_w * geo.c_swz, mapC, &sh->cfull[cs],
                               ti.d.n0 + ch * geo.c_cols, row0 + w * rows_w);
#endif
#if VB_C_NEXT_PREFETCH
            // even chunks: L2-prefetch the next chunk's sub-boxes (the adjacent 128 bytes of each row)
            if ((ch & 1) == 0 && ch + 1 < nch)
              for (int w = 2 * cid; w < 2 * cid + nsub; ++w)
                ptx::tma_prefetch_2d(mapC, ti.d.n0 + (ch + 1) * geo.c_cols, row0 + w * rows_w);
#endif
          } else {
            ptx::mbar_arrive(&sh->cfull[cs]);
          }
          advance(cs, cph, kCSlots);
        }
      }
    }
  } else {
    // ================================================================ epilogue (8 warps)
    // Warps 8+q and 12+q share TMEM lane quarter q (tile rows r0 .. r0+BY/4-1) and split each
    // chunk's columns in halves.  The pair meets on a 64-thread named barrier per chunk, then
    // warp 8+q TMA-stores the quarter's sub-box itself: no barrier spans all epilogue warps.
    const int q = warp & 3;
    const int half = (warp - 8) >> 2;
    const bool storer = half == 0;
    const uint64_t c_policy = ptx::policy_evict_first();
    (void)c_policy;
    int re = 0, cs = 0, pending = -1;
    uint32_t rph = 0, cph = 0, t = 0;
    AccRing acc_ring;
    for (;;) {
      VB_TWAIT(T_EPI_RFULL, ring_wait(re, rph));
#ifdef VB_TRACE
      const long long _head_t0 = clock64();
#endif
      const TileInfo ti = sh->ring[re];
      __syncwarp();
      if (lane == 0) ring_release(re);
      advance(re, rph, kRing);
      if (ti.d.gemm < 0) break;
      const float t_alpha = p.alpha[ti.d.gemm], t_beta = p.beta[ti.d.gemm];   // used after the accumulator wait
      const int BY = geo_BY(ti.d.geo) / (PAIR ? 2 : 1), BX = geo_BX(ti.d.geo);
      const TcGeom geo = tc_geom(BY, BX);
      const int row0 = ti.d.m0 + (int)rank * BY;     // this CTA's first row of the tile
      const uint8_t *mapC = tmaps + (size_t)ti.d.gemm * (kMapsPerGemm * 128) + MAP_C_ST * 128;
#ifdef VB_EXP_C_RMW
      const int n8 = (ti.d.N + 7) & ~7;
#else
      const int n8 = ti.d.N & ~7;                       // the store map's width
#endif
      const int units = tile_acc_units(ti.d, PAIR, SWAP);
      const int hu = split_units<PAIR>(units);                // the MMA warp's split, mirrored
      const int nent = hu ? 2 : 1;
      const int e = (int)(t % kAcc), e1 = (int)((t + 1) % kAcc);
      const uint32_t aph = (t / kAcc) & 1u, aph1 = ((t + 1) / kAcc) & 1u;
      t += (uint32_t)nent;
      int take;
      const int acc_col = acc_ring.place(units, take) * kAccUnit;
      // M = 128: tile row 32q + i lives in TMEM lane 32q + i.
      // M = 64 : tile row 16q + i lives in TMEM lane 32q + i, i < 16 (half sub-partitions).
      const int rows_w = BY / 4;
      const int r0 = q * rows_w;
      const int row = r0 + lane;
      const bool row_ok = lane < rows_w;
      const bool live = row0 + r0 < ti.d.M;             // any row of this quarter inside the GEMM
      const bool has_acc = ti.d.kblocks > 0;
      const int hcols = geo.c_cols / 2;                  // this warp's columns of a chunk
      const uint32_t tbase = tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)acc_col + half * hcols;
#ifdef VB_TRACE
      tr[T_EPI_HEAD] += clock64() - _head_t0;
#endif
      VB_TWAIT(T_EPI_TFULL, ptx::mbar_wait(&sh->tfull[e], aph));
      if (nent == 2) ptx::mbar_wait(&sh->tfull[e1], aph1);   // committed with e
      if (lane == 0) VB_STAMP(6);
      ptx::tc_fence_after();
#ifdef VB_TRACE
      const long long _tile_t0 = clock64();
#endif

      auto tload = [&](int ch, uint32_t *acc) {
        const uint32_t ta = tbase + ch * geo.c_cols;
        if (hcols == 32)
          ptx::tmem_ld_32x32b_x32(ta, *reinterpret_cast<uint32_t(*)[32]>(acc));
        else
          ptx::tmem_ld_32x32b_x16(ta, acc);
      };
      auto release_entry = [&](int ent) {              // accumulator (part) drained: hand it back early
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          if (!PAIR || leader)
            ptx::mbar_arrive(&sh->tempty[ent]);
          else   // the accumulator reads are complete (tcgen05.wait::ld) and publish no data: relaxed
            ptx::mbar_arrive_remote_relaxed(ptx::mapa(&sh->tempty[ent], 0));
        }
      };
      auto release_acc = [&]() { release_entry(e); };
      if (SWAP && (ti.d.flags & kFlagSwap)) {
        // swap-AB tile: TMEM lane 32q + i holds C column n0 + 32q + i, TMEM column j holds C row
        // m0 + j.  Warp 8+q takes rows [0, nr/2), warp 12+q rows [nr/2, nr), eight at a time;
        // every lane reads and writes one C column, so each row is one 64-byte warp access.
        const int nr = swap_rows(ti.d), hr = nr / 2, j0 = half * hr;
        const int col = ti.d.n0 + q * 32 + lane;
        const bool col_ok = col < ti.d.N;
        uint16_t *cc = static_cast<uint16_t *>(p.C[ti.d.gemm]) + (size_t)(ti.d.m0 + j0) * ti.d.ldc + col;
        const int nrow = min(hr, ti.d.M - (ti.d.m0 + j0));
        for (int jb = 0; jb < hr; jb += 8) {
          uint32_t v[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) v[j] = 0u;
          if (has_acc) {
            ptx::tmem_ld_32x32b_x8(tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc_col + j0 + jb), v);
            ptx::tmem_ld_wait();
          }
          if (jb + 8 >= hr) release_acc();             // accumulator drained
          float old[8];
#pragma unroll
          for (int j = 0; j < 8; ++j)
            old[j] = (t_beta != 0.f && col_ok && jb + j < nrow) ? c_to_float<AB_FMT>(cc[(size_t)(jb + j) * ti.d.ldc])
                                                                 : 0.f;
#pragma unroll
          for (int j = 0; j < 8; ++j)
            if (col_ok && jb + j < nrow) {
              const float a = __uint_as_float(v[j]);
              cc[(size_t)(jb + j) * ti.d.ldc] =
                  float_to_c<AB_FMT>(t_beta != 0.f ? fmaf(t_alpha, a, t_beta * old[j]) : t_alpha * a);
#ifdef VB_COVERAGE
              cov_add(cc + (size_t)(jb + j) * ti.d.ldc);
#endif
            }
        }
        continue;
      }
      auto process = [&](int ch, const uint32_t *acc) {
        const int col0 = ti.d.n0 + ch * geo.c_cols;
        VB_TWAIT(T_EPI_CFULL, ptx::mbar_wait(&sh->cfull[cs], cph));
        uint8_t *cb = cbuf + (size_t)cs * kCSlotBytes;
        {
          VB_T0();
#ifdef VB_EXP_NOMATH
          if (false) {
#else
          if (row_ok && live) {
#endif
            if (hcols == 32)
              epi_row<AB_FMT, 4>(cb, row, geo.c_swz, half * 4, acc, t_alpha, t_beta);
            else
              epi_row<AB_FMT, 2>(cb, row, geo.c_swz, half * 2, acc, t_alpha, t_beta);
          }
          VB_TADD(T_EPI_MATH);
        }
#ifdef VB_COVERAGE
        if (row_ok && live && row0 + row < ti.d.M) {   // the elements this thread's row stores
          const uint8_t *crow = static_cast<const uint8_t *>(p.C[ti.d.gemm]) + (size_t)(row0 + row) * ti.d.ldc * 2;
          for (int j = col0 + half * hcols; j < min(col0 + (half + 1) * hcols, ti.d.N); ++j) cov_add(crow + (size_t)j * 2);
        }
#endif
#if defined(VB_EXP_NOSTORE) || defined(VB_EXP_NOTAIL)
        if (false) {
#else
        if ((ti.d.flags & 1) && col0 + geo.c_cols > ti.d.N) {
#endif
          // The chunk ends inside the row's last, partial 16-byte granule (N % 8 != 0): the TMA
          // store below stops at N & ~7, and the thread that computed the granule stores its
          // N % 8 elements itself.
          const int g0 = n8 - col0;                      // granule's first column in the chunk
          const int grow = row0 + row;
          if (g0 >= half * hcols && g0 < (half + 1) * hcols && row_ok && grow < ti.d.M) {
            const uint4 w = *reinterpret_cast<const uint4 *>(cb + ptx::swz((uint32_t)(row * geo.c_swz + g0 * 2), geo.c_swz));
            uint8_t *crow = static_cast<uint8_t *>(p.C[ti.d.gemm]) + ((size_t)grow * ti.d.ldc + n8) * 2;
            // the granule is 16-byte aligned: its N % 8 elements go out as at most three stores
            // (8 + 4 + 2 bytes) -- one L2 write per store and row, not one per element
            const int nt = ti.d.N & 7;
            if (nt & 4) *reinterpret_cast<uint2 *>(crow) = make_uint2(w.x, w.y);
            if (nt & 2) *reinterpret_cast<uint32_t *>(crow + (nt & 4) * 2) = (nt & 4) ? w.z : w.x;
            if (nt & 1) {
              const int e = nt & 6;                       // the last element's index in the granule
              const uint32_t word = e >= 4 ? (e == 6 ? w.w : w.z) : (e == 2 ? w.y : w.x);
              *reinterpret_cast<uint16_t *>(crow + e * 2) = (uint16_t)(word & 0xFFFFu);
            }
          }
        }
        // TMA store of the quarter's sub-box; rows >= M and columns >= N & ~7 are clipped by the
        // TMA unit.  Every chunk commits one bulk group (possibly empty), so "all but the newest
        // group have read their smem" always covers the previous chunk's slot.
        VB_TWAIT(T_EPI_FENCEBAR, ptx::fence_proxy_async_smem(); ptx::named_bar_sync(1 + q, 64));
        VB_T0();
        if (storer && lane == 0 && ptx::elect_lane0()) {
#ifdef VB_EXP_NOSTORE
          if (false) {
#else
          if (live && col0 < n8) {
#endif
#if VB_CSTORE_HINT
            ptx::tma_store_2d_hint(mapC, cb + r0 * geo.c_swz, col0, row0 + r0, c_policy);
#else
            ptx::tma_store_2d(mapC, cb + r0 * geo.c_swz, col0, row0 + r0);
#endif
          }
          ptx::bulk_commit();
          if (pending >= 0) {
            VB_TWAIT(T_EPI_STORE, ptx::bulk_wait_read1());   // the previous store has read its slot
            ptx::mbar_arrive(&sh->cempty[pending]);
          }
          pending = cs;
        }
        VB_TADD(T_EPI_STISSUE);
        advance(cs, cph, kCSlots);
      };

      uint32_t a0[32];
      const int nch = live_chunks(geo, ti.d.N, ti.d.n0);
      if (!has_acc) {
#pragma unroll
        for (int i = 0; i < 32; ++i) a0[i] = 0u;   // K == 0: C = beta * C
      }
      for (int ch = 0; ch < nch; ++ch) {
        if (has_acc) {
          VB_TWAIT(T_EPI_TLOAD, tload(ch, a0));
          VB_TWAIT(T_EPI_TMEM, ptx::tmem_ld_wait());
        }
        if (nent == 2 && (ch + 1) * geo.c_cols == hu * kAccUnit) release_entry(e);   // first half drained
        if (ch + 1 == nch) VB_TWAIT(T_EPI_REL, release_entry(nent == 2 ? e1 : e));
        VB_TWAIT(T_EPI_PROC, process(ch, a0));
      }
#ifdef VB_TRACE
      tr[T_EPI_LOOP] += clock64() - _tile_t0;
#endif
      if (lane == 0) VB_STAMP(7);
    }
    if (storer && lane == 0) {
      ptx::bulk_wait0();
      VB_STAMP(8);
    }
  }
#ifdef VB_TRACE
  tr[T_TOTAL] = clock64() - t_start;
  if (lane == 0 && p.trace)
    for (int i = 0; i < kTraceSlots; ++i)
      if (tr[i]) atomicAdd(reinterpret_cast<unsigned long long *>(p.trace) + i, (unsigned long long)tr[i]);
#endif
  __syncwarp();
  ptx::tc_fence_before();
  if (PAIR)
    ptx::cluster_sync();   // no peer MMA / remote arrive may still target this CTA
  else
    __syncthreads();
  ptx::tc_fence_after();
  if (threadIdx.x == 0) VB_STAMP(9);
  if (warp == 1) {
    if (PAIR)
      ptx::tmem_dealloc_pair(tmem_base, kTmemCols);
    else
      ptx::tmem_dealloc(tmem_base, kTmemCols);
  }
  // The last CTA to finish resets the work-list counter, so back-to-back launches of the same
  // bound plan -- including replays of a CUDA graph that captured only vb_exec_bound -- need no
  // reset.  Every CTA made its final claim (one that returned >= n_blocks) before getting here.
  if (threadIdx.x == 0) {
    if (ptx::atom_add_acq_rel_gpu(&p.counter[1], 1) == (int)gridDim.x - 1) {
      atomicExch(&p.counter[0], 0);
      atomicExch(&p.counter[1], 0);
    }
    VB_STAMP(10);
#ifdef VB_TIMELINE_ALL
    vb_stamp_all(p.trace, 1);
#endif
  }
}

// Bind-time prep: patch the global address of every per-GEMM tensor map (A, B, C) with the
// caller's pointers (tensormap.replace), and reset the dynamic work-list counters.  The maps
// are only ever modified here, in a launch that completes before any GEMM kernel using them
// starts (stream order), so the GEMM kernel issues no per-map acquire fence (each one is a full
// scoreboard drain plus a descriptor-cache invalidate); tests re-bind one plan to alternating
// buffers to check that no stale descriptor is ever used.
__global__ void vb_tc_prep(uint8_t *tmaps, const void *const *A, const void *const *B, void *const *C,
                           const GemmParam *gemms, int batch, int32_t *counter) {
#ifndef VB_NO_PDL
  asm volatile("griddepcontrol.launch_dependents;");   // the GEMM kernel may start its setup now
#endif
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) {
    counter[0] = counter[1] = 0;   // pair kernel
    counter[2] = counter[3] = 0;   // 1-SM kernel
  }
  if (i >= batch * kMapsPerGemm) return;
  const int g = i / kMapsPerGemm, w = i % kMapsPerGemm;
  const GemmParam gp = gemms[g];
  if (gp.M <= 0 || gp.N <= 0) return;
  const int BY = (gp.row >> 8) & 0xFF;
  if (w != MAP_C && w != MAP_C_ST && gp.K <= 0) return;
  if (w == MAP_A_TAIL && gp.M % BY == 0) return;        // map not encoded
  if (w == MAP_B_TAIL && (gp.K % 64 == 0 || (gp.row & kGemmConv))) return;   // mirrors upload()
  if (w == MAP_C_ST && gp.N < 8) return;
  const void *ptr = (w == MAP_A || w == MAP_A_TAIL) ? A[g]
                    : (w == MAP_B || w == MAP_B_TAIL) ? B[g]
                                                      : static_cast<const void *>(C[g]);
  ptx::tmap_replace_address(tmaps + (size_t)i * 128, ptr);
  ptx::tmap_release();
}

}  // namespace tck

#ifdef VB_COVERAGE
VB_COV_SETTER(tc_set_coverage)
#endif

size_t tc_smem_bytes() { return tck::smem_bytes<false>(); }

cudaError_t tc_configure() {
  cudaError_t e = cudaSuccess;
  const int smem = (int)tck::smem_bytes<false>(), smem2 = (int)tck::smem_bytes<true>();
  if (e == cudaSuccess) e = cudaFuncSetAttribute(tck::vb_tc_kernel<1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(tck::vb_tc_kernel<0, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(tck::vb_tc_kernel<1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(tck::vb_tc_kernel<0, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tck::vb_tc_kernel<1, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tck::vb_tc_kernel<0, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  return e;
}

cudaError_t launch_tc_prep(uint8_t *tmaps, const void *const *A, const void *const *B, void *const *C,
                           const GemmParam *gemms, int batch, int32_t *counter, cudaStream_t stream) {
  const int n = batch * kMapsPerGemm;
  tck::vb_tc_prep<<<n > 0 ? (n + 255) / 256 : 1, 256, 0, stream>>>(tmaps, A, B, C, gemms, batch, counter);
  return cudaGetLastError();
}

// grid = persistent CTAs; pair = launch as clusters of 2 (grid must be even)
cudaError_t launch_tc(const TcArgs &args, int grid, bool bf16, bool pair, bool swap, cudaStream_t stream) {
  if (grid <= 0) return cudaSuccess;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(tck::kThreads);
  cfg.dynamicSmemBytes = pair ? tck::smem_bytes<true>() : tck::smem_bytes<false>();
  cfg.stream = stream;
  cudaLaunchAttribute attr[2];
  int na = 0;
#ifndef VB_NO_PDL
  // programmatic dependent launch: may start while the previous kernel on the stream (the
  // bind-time prep kernel) finishes; the kernel waits for it (griddepcontrol.wait) after setup
  attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[na].val.programmaticStreamSerializationAllowed = 1;
  ++na;
#endif
  if (pair) {
    attr[na].id = cudaLaunchAttributeClusterDimension;
    attr[na].val.clusterDim.x = 2;
    attr[na].val.clusterDim.y = 1;
    attr[na].val.clusterDim.z = 1;
    ++na;
  }
  cfg.attrs = attr;
  cfg.numAttrs = (unsigned)na;
  if (pair)
    return bf16 ? cudaLaunchKernelEx(&cfg, tck::vb_tc_kernel<1, true>, args)
                : cudaLaunchKernelEx(&cfg, tck::vb_tc_kernel<0, true>, args);
  if (swap)
    return bf16 ? cudaLaunchKernelEx(&cfg, tck::vb_tc_kernel<1, false, true>, args)
                : cudaLaunchKernelEx(&cfg, tck::vb_tc_kernel<0, false, true>, args);
  return bf16 ? cudaLaunchKernelEx(&cfg, tck::vb_tc_kernel<1, false>, args)
              : cudaLaunchKernelEx(&cfg, tck::vb_tc_kernel<0, false>, args);
}

}  // namespace vb
