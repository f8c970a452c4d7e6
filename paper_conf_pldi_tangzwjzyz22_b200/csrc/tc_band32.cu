// tc_band32.cu -- tensor-core kernels for fp32 window attention on sm_100a (the paper's precision:
// "f32", Fig. 8), windows with w <= 32 (halo NK = round_up(128 + 2w, 64) <= 192
// rows), d a multiple of 64 up to 512: the C2a shape of BASELINE configs[1-2].
//
// Arithmetic.  Every fp32 operand x enters the tensor cores as a pair of bf16 planes,
// hi = bf16(x) and lo = bf16(x - hi) (16 significant bits), and every product as three bf16 MMAs
// hi.hi + hi.lo + lo.hi into an fp32 TMEM accumulator; the dropped lo.lo term and the rounding of
// lo are ~2^-17 relative.  Softmax, lse, D and all accumulations stay fp32.  A simulation of this
// arithmetic on the C2a shape puts every output within 0.41 of the north_star bound (rtol 1e-4,
// atol 1e-4 max|R|); tests/test_gpu_parity.py checks the kernels element by element.  kind::tf32
// would need 3 MMAs at half the bf16 rate and K-major operands only (tools/tf32_modes_probe.cu:
// MN-major tf32 B operands are not executed), i.e. transposed copies of V, K, dO, Q for the
// output products; the bf16 planes keep the MN-major B operands of tc_band.cu.
//
// Data movement.  TMA loads fp32 box pairs into a ring slot; two converter warps then rewrite
// each row IN PLACE as its two bf16 planes: the fp32 values of a row held by the box pair (the
// same row offset of two boxes) become the bf16 hi row (over the first box) and lo row (over the
// second), which are exactly the layouts the MMAs read.  Score slices: 32 columns as two 16-column
// boxes (64-byte rows, SWIZZLE_64B) -> K-major SWIZZLE_64B planes, 40 KB per slot (128 + 192 rows),
// so the 160 KB ring holds four slices in flight; output blocks: 64 keys x 128 columns as four
// 32-column boxes (SWIZZLE_128B) -> MN-major bf16 boxes (LBO 16 KB between the two 64-column
// groups).  A slot holds fp32 and its planes in the same bytes, and the HBM bytes are those of
// the fp32 tensors: 4de + 4 per row forward, 5de + 8 / 6de + 8 per row for the two backward
// kernels (the same kernel split as tc_band.cu).
//
// One persistent kernel template, three modes; a CTA owns BM = 128 rows of one (unit, residue)
// band problem and its NK-row halo (the cached window of PAPER.md Fig. 14):
//   FWD   S = Q K_h^T -> max, exp, sum (Fig. 8 / 10 dot, dot_max, softmax, PAPER.md:215-231,
//         306-321), lse -> HBM, P (hi|lo packed over S in TMEM) ; O_c = P V_h,c per 128-column
//         chunk, scaled by 1/l.  S alternates between two TMEM regions so the next tile's score
//         GEMM runs while this tile's softmax and output GEMMs do.
//   BWDQ  S = Q K_h^T, dP = dO V_h^T; P = exp(S - lse) (recomputed from the saved lse, PAPER.md:
//         489-497); D = sum_j P dP (exact, reading R1) -> workspace; dS = P (dP - D) (hi|lo over
//         S) ; dQ_c = dS K_h,c.
//   BWDKV rows = keys (each dk / dv row has one writer, Fig. 13(d)); S^T = K Q_h^T,
//         dP^T = V dO_h^T; P^T (hi|lo over dP^T), dS^T (hi|lo over S^T); dV_c = P^T dO_h,c,
//         dK_c = dS^T Q_h,c.
//
// Roles (512 threads): warps 0-3 softmax (thread t <-> row m0 + t <-> TMEM lane t), 4-7
// epilogue (TMEM -> fp32 -> smem -> TMA store), 8 TMA producer + TMEM allocator, 9 MMA issuer,
// 10-15 converters (the conversion is latency bound per warp: 2 warps converted a 40 KB slot in
// ~4 kclk, tools/trace32.py; the softmax and epilogue work in 16-column pieces to stay within
// the 128 registers per thread of 16 warps).  TMEM: R0 = [0, 192),
// R1 = [192, 384), the output accumulator [384, 512).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <mutex>

#include "internal.h"
#include "tc_common.cuh"
#include "tile_sched.cuh"
#include "tmap.h"

namespace ftw {
namespace {

using namespace tc;

enum { FWD = 0, BWDQ = 1, BWDKV = 2 };

constexpr int BM = 128;
constexpr int KB = 64;                    // keys per output block
constexpr int CW = 128;                   // output columns per accumulation
constexpr int NST = 5;                    // ring slots
constexpr uint32_t SLOT = 40 * 1024;      // fp32 score slice (128 + 192 rows x 32 cols) / 64 x 128 block
// BWDKV with the dS tape streams no score slices: six 32 KB slots (a 96-row slice of one tape
// plane, [tsw / 4][97][4] floats with tsw <= 68, or a 64 x 128 output block), so the tape slots of
// the next operand and a whole output chunk's key blocks fit in the ring together.  No scratch.
constexpr int NST_XT = 6;
constexpr uint32_t SLOT_XT = 32 * 1024;
constexpr int TROWS = 96, TBOX = TROWS + 1;   // tape rows per slot; box rows (odd row stride: no bank conflicts)
static_assert(TBOX * 68 * 4 <= (int)SLOT_XT, "tape slot");
constexpr uint32_t STG = 32 * 128;        // one epilogue warp's 32-row x 32-col fp32 staging box
constexpr int NSTG = 1;                   // staging boxes per epilogue warp (five ring slots fit)
constexpr int NSTG_XT = 2;                // in the tape dK/dV kernel (its eight drains per tile)
constexpr int NTHREADS = 512;
constexpr int NCONV = 6;                  // converter warps
constexpr int RES_PER_LAUNCH = 8;
static_assert(RES_PER_LAUNCH <= SCHED_MAX_RES, "residue table of the tile cursor");
constexpr uint32_t R0 = 0, R1 = 192, RACC = 384;
constexpr int WMAX_SB = 64;               // steps of a WIDE tile (w <= 6080)
constexpr float RESCALE_LOG2 = 20.f;      // WIDE FWD lazy rescaling: P <= 2^20 between max moves
constexpr float LOG2E = 1.4426950408889634f;
constexpr float LN2 = 0.6931471805599453f;

// a1/b1, a2/b2: score-GEMM operands (box rows BM / NK); ob1/ob2: output-GEMM B operands (box
// rows KB); o1/o2: outputs (box rows 32).  All fp32, 32-column SWIZZLE_128B boxes.
struct Maps {
    CUtensorMap a1, b1, a2, b2, ob1, ob2, o1, o2;
    CUtensorMap tp, ts;   // BWDKV with the dS tape: the P / dS planes, 64-row boxes
};
struct Params {
    Maps maps[RES_PER_LAUNCH];
    float* lse;   // FWD: written; BWD: read
    float* D;     // BWDQ: written; BWDKV: read
    int64_t L;
    int d, w, dil, NK, nsl;
    SchedParams sc;
    int dpoll;    // BWDKV: poll D row by row (BWDQ marked its rows D_UNSET, PDL launch)
    // lse hand-off inside ft_winattn_fwd_bwd (tc_band.cu's scheme): FWD marks its lse rows
    // D_UNSET and triggers, BWDQ (PDL) and a recomputing BWDKV read lse with ld_lse_ready
    int lsepoll;
    // dS tape (ftw::DsTape, internal.h): BWDQ stores P and dS of every band entry and sets the
    // flag of each tile it finished; BWDKV (xt) loads them instead of recomputing S^T and dP^T.
    int xt, tsw;
    int64_t grows;   // tape granule stride (rows)
    uint32_t* flags;
    float* tP;
    float* tS;
    unsigned long long* trace;   // optional phase trace (ft_winattn_debug_trace), see trace32()
    // WIDE (w > 32, d = 64): a tile's 128 + 2w halo rows are visited in nsb steps of NK = 192
    // rows, step s covering halo rows [m0 - w + 192 s, m0 - w + 192 s + 192) (keys for FWD / BWDQ,
    // queries for BWDKV); each (tile, step) is one pass of this kernel's normal work, masked by
    // |i - j| <= w, with the accumulators live across the steps of a tile.
    int nsb;
    int kbw;        // WIDE: keys per output block (NK itself when one block fits a slot, else KB)
    int pdl_free;   // WIDE BWDKV launched with PDL behind BWDQ: no data dependency, waits at exit
};

// Phase trace (profiling only): per CTA, clock64 stamps of its first TR_SLOTS slots --
// [0] producer issued the TMA, [1] converter started, [2] converter done, [3] MMA issue start,
// [4] MMA issue end -- and of its first TR_TILES tiles at [TR_SLOTS * 5 + tile * 16 + e]:
// 0 softmax s_full seen, 1 softmax p_full arrived, 2.. epilogue o_full seen per accumulation.
constexpr int TR_SLOTS = 96, TR_TILES = 4, TR_PER_CTA = TR_SLOTS * 5 + TR_TILES * 16;
__device__ __forceinline__ void trace_slot(const Params& p, int k, int e) {
    if (p.trace && k < TR_SLOTS) p.trace[(size_t)blockIdx.x * TR_PER_CTA + k * 5 + e] = clock64();
}
__device__ __forceinline__ void trace_tile(const Params& p, int j, int e) {
    if (p.trace && j < TR_TILES && e < 16) p.trace[(size_t)blockIdx.x * TR_PER_CTA + TR_SLOTS * 5 + j * 16 + e] = clock64();
}

constexpr size_t SCRATCH = 3 * 128 * 4 + 2 * 192 * 4;   // FWD row 1/l [3][128]; BWDKV column lse / D
constexpr size_t BAR_BYTES = 512;
constexpr size_t SMEM_BYTES = 1024 + NST * SLOT + 4 * NSTG * STG + SCRATCH + BAR_BYTES;
constexpr size_t SMEM_BYTES_XT = 1024 + NST_XT * SLOT_XT + 4 * NSTG_XT * STG + BAR_BYTES;
static_assert(SMEM_BYTES <= 227 * 1024 && SMEM_BYTES_XT <= 227 * 1024, "shared memory plan");
static_assert(3 * NST_XT * 8 + 16 * 8 + 4 <= BAR_BYTES, "barrier area");

using Tile = SchedTile;
using TileCursor = SchedCursor<BM>;

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
// x -> (bf16(x), bf16(x - bf16(x))) for two values, packed as bf16x2 words
__device__ __forceinline__ void split2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    hi = pack_bf16x2(x0, x1);   // RN; x0 in the low half
    lo = pack_bf16x2(x0 - __uint_as_float(hi << 16), x1 - __uint_as_float(hi & 0xFFFF0000u));
}
__device__ __forceinline__ int chunk_w(int d, int c) { return d - CW * c < CW ? d - CW * c : CW; }
__device__ __forceinline__ bool band_ok(int n, int t, int w, int mcol, int Lr) {
    return (unsigned)(n - t) <= (unsigned)(2 * w) && mcol >= 0 && mcol < Lr;
}

// In-place fp32 -> bf16 hi / lo planes of box pairs: a pair is box0 at p and box1 at p + R * RB,
// RB-byte rows (RB = 128: 32 fp32 per box row, SWIZZLE_128B, 16-byte granule g of row r at
// (g ^ (r & 7)) * 16; RB = 64: 16 fp32, SWIZZLE_64B, granule g at (g ^ ((r >> 1) & 3)) * 16).
// The 2 RB / 4 fp32 of row r (box0 columns first) become the bf16 hi row over box0 and the lo row
// over box1 -- the K-major (score slices) or MN-major (output blocks) bf16 operand rows.  One
// thread converts a whole row: it reads every byte it writes, so no thread waits for another
// (the earlier four-threads-per-row form needed a __syncwarp between reads and writes and ran
// ~5.6 instructions per element; this one ~2, tools/trace32.py: 1.8 -> see DESIGN.md §7).  The
// rows of two pairs (R0 rows at p0, R1 rows at p1) are dealt round robin to the 32 NCONV
// converter threads; ct: converter thread 0 .. 32 NCONV - 1.
template <int RB>
__device__ __forceinline__ int swz(int g, int r) { return RB == 128 ? (g ^ (r & 7)) : (g ^ ((r >> 1) & 3)); }

// (x0, x1) -> hi = bf16x2 RN, lo = bf16x2 RN of (x0, x1) - hi, with one packed fp32 subtraction
__device__ __forceinline__ void split2p(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    asm("{\n\t.reg .b32 h0, h1, r0, r1;\n\t.reg .b64 xx, hh, rr;\n\t"
        "cvt.rn.bf16x2.f32 %0, %3, %2;\n\t"
        "shl.b32 h0, %0, 16;\n\tand.b32 h1, %0, 0xffff0000;\n\t"
        "mov.b64 xx, {%2, %3};\n\tmov.b64 hh, {h0, h1};\n\t"
        "sub.rn.f32x2 rr, xx, hh;\n\t"
        "mov.b64 {r0, r1}, rr;\n\t"
        "cvt.rn.bf16x2.f32 %1, r1, r0;\n\t}"
        : "=r"(hi), "=r"(lo)
        : "f"(x0), "f"(x1));
}

template <int RB>
__device__ __forceinline__ void convert_rows2(uint8_t* p0, int R0, uint8_t* p1, int R1, int ct) {
    constexpr int NX = RB / 16;   // 16-byte fp32 granules per box row
    for (int vr = ct; vr < R0 + R1; vr += 32 * NCONV) {
        const bool first = vr < R0;
        uint8_t* p = first ? p0 : p1;
        const int R = first ? R0 : R1, r = first ? vr : vr - R0;
        uint4 v[2 * NX];
#pragma unroll
        for (int b = 0; b < 2; ++b)
#pragma unroll
            for (int g = 0; g < NX; ++g)
                v[b * NX + g] = *reinterpret_cast<const uint4*>(p + b * R * RB + r * RB + (swz<RB>(g, r) << 4));
#pragma unroll
        for (int G = 0; G < NX; ++G) {   // output granule G: fp32 columns 8G .. 8G + 7
            const uint4 a = v[2 * G], c = v[2 * G + 1];
            uint32_t hi[4], lo[4];
            split2p(__uint_as_float(a.x), __uint_as_float(a.y), hi[0], lo[0]);
            split2p(__uint_as_float(a.z), __uint_as_float(a.w), hi[1], lo[1]);
            split2p(__uint_as_float(c.x), __uint_as_float(c.y), hi[2], lo[2]);
            split2p(__uint_as_float(c.z), __uint_as_float(c.w), hi[3], lo[3]);
            const uint32_t off = r * RB + (swz<RB>(G, r) << 4);
            *reinterpret_cast<uint4*>(p + off) = make_uint4(hi[0], hi[1], hi[2], hi[3]);
            *reinterpret_cast<uint4*>(p + R * RB + off) = make_uint4(lo[0], lo[1], lo[2], lo[3]);
        }
    }
}

// K-major SWIZZLE_64B smem descriptor (64-byte rows; SBO = 8 rows x 64 B)
__device__ __forceinline__ uint64_t sdesc_sw64(uint32_t saddr) {
    uint64_t desc = 0;
    desc |= (uint64_t)((saddr >> 4) & 0x3FFFu);
    desc |= (uint64_t)1 << 16;
    desc |= (uint64_t)(512u >> 4) << 32;
    desc |= (uint64_t)1 << 46;   // version (sm_100)
    desc |= (uint64_t)4 << 61;   // SWIZZLE_64B
    return desc;
}

// The slot sequence every role walks in the same order.  FWD: G(0), then per tile j: G(j+1),
// O(j).  BWD: per tile: G(j), O(j).  G = nsl score slices (BWD: two slots per slice, S then dP);
// O = nacc accumulations x nkb key blocks.
template <int MODE>
struct Seq {
    static constexpr int NA = MODE == FWD ? 1 : 2;
    static constexpr int NOUT = MODE == BWDKV ? 2 : 1;
};

// use counts of the three accumulator regions (registers, no dynamic indexing)
struct AccUses {
    int u0 = 0, u1 = 0, u2 = 0;
    __device__ __forceinline__ int get(int r) const { return r == 0 ? u0 : r == 1 ? u1 : u2; }
    __device__ __forceinline__ void inc(int r) {
        if (r == 0) ++u0;
        else if (r == 1) ++u1;
        else ++u2;
    }
};

// XT: the dS tape (BWDQ writes it, BWDKV reads it) as its own instantiation, so neither kernel's
// instruction working set carries the other path's code (p.xt is set iff XT)
template <int MODE, bool WIDE, bool XT>
__global__ void __launch_bounds__(NTHREADS, 1) tc_band32_kernel(const __grid_constant__ Params p) {
    static_assert(!XT || (MODE != FWD && !WIDE), "tape instantiations: band BWDQ / BWDKV only");
    using C = Seq<MODE>;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int NK = p.NK, nsl = p.nsl, w = p.w, d = p.d;
    const int kbw = WIDE ? p.kbw : KB;        // keys per output block
    const int nkb = NK / kbw, nch = NK / 32;
    const int ncw = (d + CW - 1) / CW;      // output chunks per tensor (the last may be 64 wide)
    const int nacc = ncw * C::NOUT;         // accumulations per tile
    const int nsb = WIDE ? p.nsb : 1;       // sub-bands per tile
    // WIDE backward: the epilogue warps also run the softmax (column halves; no row reduction
    // there), so each step's softmax takes about half as long
    constexpr bool SPLITSM = WIDE && MODE != FWD;
    // TMEM: R0 = [0, NK), R1 = [r1, r1 + NK), accumulators from racc.  WIDE d = 128 uses 128-row
    // steps (R1 at 128, the accumulators at 256: BWDKV's dV and dK take 128 columns each).
    const uint32_t r1 = WIDE ? (d == 128 ? 128u : (uint32_t)NK) : R1;
    const uint32_t racc = (WIDE && d == 128) ? 256u : RACC;
    // first halo row of step sb relative to m0 (normal mode: -w)
    auto koff = [&](int sb) -> int { return WIDE ? -w + (int)NK * sb : -w; };

    if (MODE == BWDQ && XT) {   // clear this CTA's tile flags before BWDKV may launch
        TileCursor cr(p.sc);
        Tile T;
        while (cr.next(p.sc, T))
            if (threadIdx.x == 0) p.flags[(int64_t)T.u * p.L + T.r + (int64_t)T.m0 * p.dil] = 0u;
        __threadfence();
        __syncthreads();
    } else if (MODE == BWDQ && p.dpoll) {   // mark this CTA's D rows unset before BWDKV may launch
        TileCursor cr(p.sc);
        Tile T;
        while (cr.next(p.sc, T)) {
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            for (int i = threadIdx.x; i < BM && T.m0 + i < T.Lr; i += NTHREADS)
                reinterpret_cast<uint32_t*>(p.D)[rowbase + (int64_t)(T.m0 + i) * p.dil] = D_UNSET;
        }
        __threadfence();
        __syncthreads();
    }
    if (MODE == FWD && p.lsepoll) {   // lse rows unset, then let the dQ kernel (PDL) launch
        TileCursor cr(p.sc);
        Tile T;
        while (cr.next(p.sc, T)) {
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            for (int i = threadIdx.x; i < BM && T.m0 + i < T.Lr; i += NTHREADS)
                reinterpret_cast<uint32_t*>(p.lse)[rowbase + (int64_t)(T.m0 + i) * p.dil] = D_UNSET;
        }
        __threadfence();
        __syncthreads();
    }
    if (MODE == BWDQ || (MODE == FWD && p.lsepoll)) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");

    constexpr bool xt = MODE == BWDKV && XT;
    const int nst = xt ? NST_XT : NST;
    const uint32_t slotb = xt ? SLOT_XT : SLOT;
    uint8_t* slots = smem;
    const int nstg = xt ? NSTG_XT : NSTG;
    uint8_t* stg = smem + nst * slotb;                                  // [4 warps][nstg] fp32 boxes
    float* scratch = reinterpret_cast<float*>(stg + 4 * nstg * STG);
    float* rowScale = scratch;                                          // FWD [3][128]
    float* colLse = scratch + 3 * 128;                                  // BWDKV [192] lse * log2e
    float* colD = colLse + 192;                                         // BWDKV [192]
    uint64_t* bars = reinterpret_cast<uint64_t*>(reinterpret_cast<uint8_t*>(scratch) + (xt ? 0 : SCRATCH));
    uint64_t* full = bars;                // [nst] TMA bytes landed
    uint64_t* conv = bars + NST_XT;       // [nst] planes written (4 converter warps)
    uint64_t* empty = bars + 2 * NST_XT;  // [nst] MMAs done with the slot
    uint64_t* s_full = bars + 3 * NST_XT; // [2] score GEMMs of a tile done (FWD: region j & 1)
    uint64_t* p_full = s_full + 2;     // [2] softmax wrote the MMA operands of a tile (4 warps)
    uint64_t* o_full = s_full + 4;     // [3] accumulation done, per accumulator region (acc_rid)
    uint64_t* o_empty = s_full + 7;    // [3] accumulator drained (4 epilogue warps)
    // xt: [0] R1 free (the tile's last dK accumulation in R1 drained), [1] R0 free (last dV one in
    // R0): one phase per tile each, so the softmax warps never lag two phases behind (o_empty
    // completes u0 times per tile and is waited only by the MMA issuer, use by use)
    uint64_t* xfree = s_full + 10;
    uint64_t* pv_done = s_full + 12;  // WIDE FWD [2]: the output GEMMs of step k done (parity k & 1)
    uint64_t* rs_full = s_full + 14;  // WIDE FWD [2]: 1/l and lse of tile j published (4 warps)
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 16);
    // Accumulator of accumulation a: RACC, except in BWDKV with the dS tape, where the dV (dK)
    // chunks alternate between R0 (R1) and RACC, ending on RACC: during dV R1 holds the A operand
    // P^T and R0 is free (dS^T is built into it after the last R0 drain), during dK R0 holds dS^T
    // and R1 is free -- so an accumulation runs while the epilogue drains the previous one.
    auto acc_rid = [&](int a) -> int {
        if (WIDE) return a;   // FWD / BWDQ: one accumulation; BWDKV: dV (0), dK (1), both live across sub-bands
        if (!xt || ((ncw - 1 - a % ncw) & 1) == 0) return 0;
        return a < ncw ? 1 : 2;
    };
    // (the R1 accumulator sits at column 256, 128-aligned like the others)
    auto acc_col = [&](int rid) -> uint32_t {
        if (WIDE) return racc + (uint32_t)d * rid;
        return rid == 0 ? RACC : rid == 1 ? R0 : R1 + 64;
    };
    const int npl = (NK + TROWS - 1) / TROWS;   // tape slots per plane
    // (with ncw >= 2, the host's condition for xt, the last R0 / R1 accumulation is chunk ncw - 2)

    if (warp == 8) {
        if (lane == 0) {
            for (int i = 0; i < nst; ++i) {
                mbar_init(&full[i], 1);
                mbar_init(&conv[i], NCONV);
                mbar_init(&empty[i], 1);
            }
            for (int i = 0; i < 2; ++i) {
                mbar_init(&s_full[i], 1);
                mbar_init(&p_full[i], SPLITSM ? 8 : 4);
            }
            for (int i = 0; i < 3; ++i) {
                mbar_init(&o_full[i], 1);
                mbar_init(&o_empty[i], 4);
            }
            mbar_init(&xfree[0], 4);
            mbar_init(&xfree[1], 4);
            for (int i = 0; i < 2; ++i) {
                mbar_init(&pv_done[i], 1);
                mbar_init(&rs_full[i], 4);
            }
            fence_barrier_init();
            for (int i = 0; i < p.sc.nr; ++i) {
                const Maps& mp = p.maps[i];
                tma_prefetch(&mp.a1); tma_prefetch(&mp.b1); tma_prefetch(&mp.ob1); tma_prefetch(&mp.o1);
                if (C::NA == 2) { tma_prefetch(&mp.a2); tma_prefetch(&mp.b2); }
                if (C::NOUT == 2) { tma_prefetch(&mp.ob2); tma_prefetch(&mp.o2); }
            }
        }
        __syncwarp();
        tmem_alloc(tmem_holder, 512);
        tmem_relinquish();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tbase = *tmem_holder;

    // ------------------------------------------------------------------ shared slot walker
    // fn(kind, T, a, b): kind 0 = score slot (slice a, operand pair b = 0 S / 1 dP), 1 = output
    // block (accumulation a, key block b).  Called in slot order.
    auto walk = [&](auto&& fn) {
        TileCursor cg(p.sc), co(p.sc);
        Tile Tg, To;
        bool hg = cg.next(p.sc, Tg);
        if constexpr (WIDE) {
            // steps (tile, sub-band); FWD: G(step 0), then per step G(step + 1), O(step); BWD: G, O
            if (MODE == FWD) {
                int sg = 0;
                auto gnext = [&]() {
                    for (int s = 0; s < nsl; ++s) fn(0, Tg, s, 0, sg);
                    if (++sg == nsb) {
                        sg = 0;
                        hg = cg.next(p.sc, Tg);
                    }
                };
                if (hg) gnext();
                while (co.next(p.sc, To))
                    for (int so = 0; so < nsb; ++so) {
                        if (hg) gnext();
                        for (int a = 0; a < nacc; ++a)
                            for (int kb = 0; kb < nkb; ++kb) fn(1, To, a, kb, so);
                    }
            } else {
                while (co.next(p.sc, To))
                    for (int so = 0; so < nsb; ++so) {
                        for (int s = 0; s < nsl; ++s) {
                            fn(0, To, s, 0, so);
                            fn(0, To, s, 1, so);
                        }
                        for (int a = 0; a < nacc; ++a)
                            for (int kb = 0; kb < nkb; ++kb) fn(1, To, a, kb, so);
                    }
            }
            return;
        }
        if (MODE == FWD) {
            if (hg) {
                for (int s = 0; s < nsl; ++s) fn(0, Tg, s, 0, 0);
                hg = cg.next(p.sc, Tg);
            }
            while (co.next(p.sc, To)) {
                if (hg) {
                    for (int s = 0; s < nsl; ++s) fn(0, Tg, s, 0, 0);
                    hg = cg.next(p.sc, Tg);
                }
                for (int a = 0; a < nacc; ++a)
                    for (int kb = 0; kb < nkb; ++kb) fn(1, To, a, kb, 0);
            }
        } else if (xt) {
            // Tape slots (npl of 128 rows per plane) sit one output chunk ahead of their use, so
            // an operand is built while the last chunk of the other output accumulates:
            //   P(0); per tile j: dV c0 .. c[ncw-2], dS(j), dV c[ncw-1], dK c0 .. c[ncw-2],
            //   P(j+1) (if any), dK c[ncw-1].   Slot positions: xt_pos_P / xt_pos_S below.
            bool has = co.next(p.sc, To);
            if (has)
                for (int b = 0; b < npl; ++b) fn(2, To, b, 0, 0);
            while (has) {
                Tile Tnext;
                const bool hnext = co.next(p.sc, Tnext);
                auto blocks = [&](int a) {
                    for (int kb = 0; kb < nkb; ++kb) fn(1, To, a, kb, 0);
                };
                for (int a = 0; a < ncw - 1; ++a) blocks(a);
                for (int b = 0; b < npl; ++b) fn(2, To, b, 1, 0);
                blocks(ncw - 1);
                for (int a = ncw; a < nacc - 1; ++a) blocks(a);
                if (hnext)
                    for (int b = 0; b < npl; ++b) fn(2, Tnext, b, 0, 0);
                blocks(nacc - 1);
                To = Tnext;
                has = hnext;
            }
        } else {
            while (co.next(p.sc, To)) {
                for (int s = 0; s < nsl; ++s) {
                    fn(0, To, s, 0, 0);
                    fn(0, To, s, 1, 0);
                }
                for (int a = 0; a < nacc; ++a)
                    for (int kb = 0; kb < nkb; ++kb) fn(1, To, a, kb, 0);
            }
        }
    };

    // ------------------------------------------------------------------ drain of one tile
    // Epilogue warps 4-7 (TMEM lanes 32 (warp - 4) ..): every accumulation of tile T -> fp32 ->
    // staging box -> TMA store, scaled by `scale` (FWD: 1/l of the row).
    auto drain_tile = [&](const Tile& T, int j, int& sidx, AccUses& uses, float scale) {
        const int ew = warp - 4;
        const uint32_t tlane = tbase + ((uint32_t)(ew * 32) << 16);
        uint8_t* mystg = stg + ew * nstg * STG;
        const Maps& mp = p.maps[T.rl];
        for (int a = 0; a < nacc; ++a) {
            const int c = C::NOUT == 2 ? a % ncw : a;
            const CUtensorMap* om = (C::NOUT == 2 && a < ncw) ? &mp.o2 : &mp.o1;   // BWDKV: dV first
            const int ngrp = chunk_w(d, c) / 32;
            const int rid = acc_rid(a);
            const uint32_t trow = tlane + acc_col(rid);
            mbar_wait(&o_full[rid], (uint32_t)uses.get(rid) & 1u);
            uses.inc(rid);
            tc_fence_after();
            if (ew == 0 && lane == 0) trace_tile(p, j, 2 + a);
            // two rounds of 64 columns (register budget of 16 warps); the accumulator is
            // released once the last columns are in registers
#pragma unroll
            for (int x = 0; x < 4; ++x) {
                if (x >= ngrp) break;
                uint32_t ov[1][32];
                tmem_ld32(trow + 32 * x, ov[0]);
                tmem_wait_ld();
                if (x == ngrp - 1) {
                    tc_fence_before();
                    warp_arrive(&o_empty[rid]);
                    if (xt && a % ncw == ncw - 2) warp_arrive(&xfree[a < ncw ? 1 : 0]);
                }
                uint8_t* sb = mystg + (sidx % nstg) * STG;
                if (lane == 0 && sidx >= nstg) {
                    if (nstg == 2) tma_store_wait_read<1>();
                    else tma_store_wait_read<0>();
                }
                __syncwarp();
#pragma unroll
                for (int g = 0; g < 8; ++g) {
                    uint4 val;
                    val.x = __float_as_uint(__uint_as_float(ov[0][4 * g + 0]) * scale);
                    val.y = __float_as_uint(__uint_as_float(ov[0][4 * g + 1]) * scale);
                    val.z = __float_as_uint(__uint_as_float(ov[0][4 * g + 2]) * scale);
                    val.w = __float_as_uint(__uint_as_float(ov[0][4 * g + 3]) * scale);
                    *reinterpret_cast<uint4*>(sb + lane * 128 + ((g ^ (lane & 7)) << 4)) = val;
                }
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) {
                    tma_store_3d(om, sb, CW * c + 32 * x, T.m0 + 32 * ew, T.u);
                    tma_store_commit();
                }
                ++sidx;
            }
        }
    };

    if (warp == 8) {
        if (lane == 0) {   // -------------------------------------------------- TMA producer
            int st = 0, k = 0;
            uint32_t ph = 0;
            walk([&](int kind, const Tile& T, int a, int b, int sb) {
                mbar_wait(&empty[st], ph ^ 1u);
                trace_slot(p, k++, 0);
                uint8_t* sp = slots + (size_t)st * slotb;
                const Maps& mp = p.maps[T.rl];
                if (kind == 2) {   // dS tape: query rows [96 a, 96 a + 97) of plane b (P, dS)
                    if (a == 0 && b == 0 && p.dpoll) {   // BWDQ may still run: wait for these rows' tiles
                        const int64_t rowbase = (int64_t)T.u * p.L + T.r;
                        const int lo = max(0, T.m0 - w) / BM, hi = min(T.Lr - 1, T.m0 + BM - 1 + w) / BM;
                        for (int tq = lo; tq <= hi; ++tq) wait_flag(p.flags + rowbase + (int64_t)tq * BM * p.dil);
                        asm volatile("fence.proxy.async.global;" ::: "memory");
                    }
                    mbar_arrive_expect_tx(&full[st], (uint32_t)(TBOX * p.tsw * 4));
                    tma_load_4d(sp, b ? &mp.ts : &mp.tp, &full[st], 0, T.m0 - w + TROWS * a, T.u, 0);
                } else if (kind == 0) {   // 32 columns: two 16-column boxes of each operand
                    const CUtensorMap* ma = b ? &mp.a2 : &mp.a1;
                    const CUtensorMap* mb = b ? &mp.b2 : &mp.b1;
                    mbar_arrive_expect_tx(&full[st], (uint32_t)(2 * BM + 2 * NK) * 64u);
                    for (int h = 0; h < 2; ++h) {
                        tma_load_3d(sp + h * BM * 64, ma, &full[st], 32 * a + 16 * h, T.m0, T.u);
                        tma_load_3d(sp + 2 * BM * 64 + h * NK * 64, mb, &full[st], 32 * a + 16 * h, T.m0 + koff(sb), T.u);
                    }
                } else {
                    const int c = C::NOUT == 2 ? a % ncw : a;
                    const int nbox = chunk_w(d, c) / 32;
                    const CUtensorMap* m = (C::NOUT == 2 && a >= ncw) ? &mp.ob2 : &mp.ob1;
                    mbar_arrive_expect_tx(&full[st], (uint32_t)nbox * kbw * 128u);
                    for (int x = 0; x < nbox; ++x)
                        tma_load_3d(sp + x * kbw * 128, m, &full[st], CW * c + 32 * x, T.m0 + koff(sb) + kbw * b, T.u);
                }
                if (++st == nst) { st = 0; ph ^= 1u; }
            });
        }
    } else if (warp >= 10) {   // ------------------------------------------------- converters
        const int ct = threadIdx.x - 320;   // 0 .. 32 NCONV - 1
        int st = 0, k = 0;
        uint32_t ph = 0;
        walk([&](int kind, const Tile&, int a, int, int) {
            mbar_wait(&full[st], ph);
            if (ct == 0) trace_slot(p, k, 1);
            uint8_t* sp = slots + (size_t)st * slotb;
            if (kind == 2) {
                // tape slot: read as fp32 by the softmax warps (arrive only, keeping the phases)
            } else if (kind == 0) {
                convert_rows2<64>(sp, BM, sp + 2 * BM * 64, NK, ct);
            } else {
                const bool full_chunk = chunk_w(d, C::NOUT == 2 ? a % ncw : a) == CW;
                convert_rows2<128>(sp, kbw, sp + 2 * kbw * 128, full_chunk ? kbw : 0, ct);
            }
            fence_proxy_async_smem();
            warp_arrive(&conv[st]);
            if (ct == 0) trace_slot(p, k, 2);
            ++k;
            if (++st == nst) { st = 0; ph ^= 1u; }
        });
    } else if (warp == 9) {
        if (lane == 0) {   // ------------------------------------------------------ MMA issuer
            const uint32_t idS = idesc_bf16(BM, NK, false, false);
            const uint32_t idO = idesc_bf16(BM, CW, false, true);
            const uint32_t idO64 = idesc_bf16(BM, 64, false, true);   // a 64-column last chunk
            int st = 0, k = 0;
            AccUses uses;   // accumulations per region so far
            uint32_t ph = 0;
            int jg = 0;          // score GEMMs: tile (WIDE: step) counter
            int jo = 0;          // output GEMMs: tile (WIDE: step) counter
            walk([&](int kind, const Tile&, int a, int b, int sb) {
                const uint32_t sa = smem_u32(slots + (size_t)st * slotb);
                if (kind == 2) {   // tape slot: no MMA (the softmax warps free it)
                    mbar_wait(&conv[st], ph);
                } else if (kind == 0) {
                    // FWD: S(jg) into region jg & 1; BWD: S into R0, dP into R1
                    const uint32_t dst = tbase + (MODE == FWD ? ((jg & 1) ? r1 : R0) : (b ? r1 : R0));
                    if (MODE != FWD && a == 0 && b == 0 && jg > 0) {
                        // R1 (dP) is free once the softmax of the previous tile read it (p_full);
                        // R0 (dS) once the previous tile's output MMAs read it (issue order)
                        mbar_wait(&p_full[(jg - 1) & 1], ((jg - 1) >> 1) & 1);
                        tc_fence_after();
                    }
                    mbar_wait(&conv[st], ph);
                    tc_fence_after();
                    trace_slot(p, k, 3);
                    const uint32_t ahi = sa, alo = sa + BM * 64, bhi = sa + 2 * BM * 64, blo = bhi + NK * 64;
#pragma unroll
                    for (int kk = 0; kk < 2; ++kk) {
                        const uint64_t dah = sdesc_sw64(ahi + kk * 32), dal = sdesc_sw64(alo + kk * 32);
                        const uint64_t dbh = sdesc_sw64(bhi + kk * 32), dbl = sdesc_sw64(blo + kk * 32);
                        mma_ss(dst, dah, dbh, idS, (a | kk) != 0);
                        mma_ss(dst, dah, dbl, idS, 1);
                        mma_ss(dst, dal, dbh, idS, 1);
                    }
                    mma_commit(&empty[st]);
                    if (a == nsl - 1 && b == C::NA - 1) {
                        mma_commit(&s_full[MODE == FWD ? (jg & 1) : 0]);
                        ++jg;
                    }
                } else {
                    // output block b of accumulation a of tile jo.  A: packed hi | lo operand in TMEM
                    // (FWD: P over S(jo); BWDQ: dS over S; BWDKV: P^T over dP^T (dV), dS^T over S^T (dK))
                    if (b == 0 && (a == 0 || (xt && a == ncw))) {   // xt: P^T (dV), dS^T (dK) built
                        if (xt) mbar_wait(&p_full[a == 0 ? 0 : 1], (uint32_t)jo & 1u);
                        else mbar_wait(&p_full[jo & 1], (jo >> 1) & 1);
                        tc_fence_after();
                    }
                    const int rid = acc_rid(a);
                    // WIDE: the accumulators live across the sub-bands of a tile
                    const bool first_sb = !WIDE || sb == 0, last_sb = !WIDE || sb == nsb - 1;
                    if (b == 0 && first_sb && uses.get(rid) > 0) {
                        mbar_wait(&o_empty[rid], (uint32_t)(uses.get(rid) - 1) & 1u);
                        tc_fence_after();
                    }
                    const uint32_t Dacc = tbase + acc_col(rid);
                    const uint32_t Areg = tbase + (MODE == FWD ? ((jo & 1) ? r1 : R0)
                                                   : (MODE == BWDKV && a < ncw) ? r1 : R0);
                    const uint32_t id = chunk_w(d, C::NOUT == 2 ? a % ncw : a) == CW ? idO : idO64;
                    mbar_wait(&conv[st], ph);
                    tc_fence_after();
                    trace_slot(p, k, 3);
                    const int kpb = kbw / 16;   // 16-key steps per output block
#pragma unroll 4
                    for (int kk = 0; kk < kpb; ++kk) {
                        const int g = kpb * b + kk;   // 16-key step over the halo
                        const uint32_t tA = Areg + 16u * g;   // hi words; lo words at + 8
                        const uint64_t dbh = sdesc_sw128(sa + kk * 2048, 2 * kbw * 128, 1024);
                        const uint64_t dbl = sdesc_sw128(sa + kbw * 128 + kk * 2048, 2 * kbw * 128, 1024);
                        mma_ts(Dacc, tA, dbh, id, !first_sb || g != 0);
                        mma_ts(Dacc, tA, dbl, id, 1);
                        mma_ts(Dacc, tA + 8, dbh, id, 1);
                    }
                    mma_commit(&empty[st]);
                    if (b == nkb - 1) {
                        if (last_sb) {
                            mma_commit(&o_full[rid]);
                            uses.inc(rid);
                        }
                        if (WIDE && MODE == FWD) mma_commit(&pv_done[jo & 1]);   // rescale hand-off
                        if (a == nacc - 1) ++jo;
                    }
                }
                trace_slot(p, k++, 4);
                if (++st == nst) { st = 0; ph ^= 1u; }
            });
        }
    } else if (warp < 4 || (SPLITSM && warp < 8)) {   // -------------------------- softmax warps
        // SPLITSM: warps 4-7 take the upper half of every row's chunks and drain the tile after its
        // last step (they are the epilogue warps)
        const int hsm = SPLITSM ? warp / 4 : 0, wq = warp % 4;
        const int t = wq * 32 + lane;
        const uint32_t lane_off = (uint32_t)(wq * 32) << 16;
        // chunks holding any band column of this warp's rows: [32 warp, 32 warp + 31 + 2w]
        const int c_lo = wq, c_hi = min(nch - 1, (32 * wq + 31 + 2 * w) / 32);
        uint32_t zero16[16];
#pragma unroll
        for (int e = 0; e < 16; ++e) zero16[e] = 0u;
        TileCursor cur(p.sc);
        Tile T;
        int j = 0;
        if (MODE == BWDKV && !p.dpoll && !p.pdl_free) asm volatile("griddepcontrol.wait;" ::: "memory");
        if constexpr (WIDE) {
            // One (tile, step) at a time.  FWD: online softmax over the steps with
            // lazy rescaling (the running max m only moves when a step's max exceeds it by more
            // than 2^RESCALE_LOG2; then this row's O partial in TMEM and l are scaled by 2^(m_old -
            // m_new) after the previous step's output GEMMs completed).  BWDQ / BWDKV: the global lse
            // and D (= dout . out, computed before the launch) make every step independent.
            int k = 0, sidx = 0;
            AccUses euses;   // SPLITSM drainers (warps 4-7)
            float m_run = 0.f, l_run = 0.f;
            bool m_set = false;   // FWD: the row has met a band entry (m_run is one of its scores)
            while (cur.next(p.sc, T)) {
                const int Lr = T.Lr, m0 = T.m0, mrow = m0 + t;
                const int64_t rowbase = (int64_t)T.u * p.L + T.r;
                const bool rowv = mrow < Lr;
                float lse2 = 0.f, Drow = 0.f;
                if (MODE == BWDQ && rowv) {
                    lse2 = p.lse[rowbase + (int64_t)mrow * p.dil] * LOG2E;
                    Drow = p.D[rowbase + (int64_t)mrow * p.dil];
                }
                for (int sb = 0; sb < nsb; ++sb, ++k) {
                    // column n of row t is in the band iff n - t + sh in [0, 2w] (halo row kb + n)
                    const int sh = NK * sb, kb = m0 + koff(sb), W2 = 2 * w;
                    const int nlo = 32 * wq - sh, nhi = 32 * wq + 31 - sh + W2;
                    const int clo = nlo > 0 ? nlo / 32 : 0, chi = nhi < 0 ? -1 : min(nch - 1, nhi / 32);
                    // chunks this warp handles: all (FWD), or its half of [clo, chi] plus the zero
                    // chunks on its side (SPLITSM)
                    const int cm = (clo + chi + 1) >> 1;
                    auto mine = [&](int c) { return !SPLITSM || (hsm == 0 ? c < cm : c >= cm); };
                    if (MODE == BWDKV) {   // lse / D of this step's halo queries
                        constexpr int NSMT = SPLITSM ? 256 : 128;
                        named_bar_sync(1, NSMT);
                        for (int n = hsm * 128 + t; n < NK; n += NSMT) {
                            const int mc = kb + n;
                            const bool ok = mc >= 0 && mc < Lr;
                            colLse[n] = ok ? p.lse[rowbase + (int64_t)mc * p.dil] * LOG2E : 0.f;
                            colD[n] = ok ? p.D[rowbase + (int64_t)mc * p.dil] : 0.f;
                        }
                        named_bar_sync(1, NSMT);
                    }
                    mbar_wait(&s_full[MODE == FWD ? (k & 1) : 0], MODE == FWD ? ((k >> 1) & 1) : (k & 1));
                    tc_fence_after();
                    const uint32_t rS = tbase + lane_off + (MODE == FWD && (k & 1) ? r1 : R0);
                    const uint32_t rP = tbase + lane_off + r1;
                    if (MODE == FWD) {
                        float cm = -INFINITY;
                        for (int c = clo; c <= chi; ++c) {
                            uint32_t rr[32];
                            tmem_ld32(rS + c * 32, rr);
                            tmem_wait_ld();
#pragma unroll
                            for (int e = 0; e < 32; ++e)
                                if ((unsigned)(c * 32 + e - t + sh) <= (unsigned)W2 && kb + c * 32 + e >= 0 && kb + c * 32 + e < Lr)
                                    cm = fmaxf(cm, __uint_as_float(rr[e]));
                        }
                        const float cms = cm * LOG2E;
                        float fac = 1.f;
                        bool need = false;
                        if (sb == 0) {
                            m_set = false;
                            m_run = 0.f;
                            l_run = 0.f;
                        }
                        if (!m_set) {   // O and l of this row are still 0: take this step's max
                            if (cm != -INFINITY) {
                                m_run = cms;
                                m_set = true;
                            }
                        } else if (cm != -INFINITY && cms > m_run + RESCALE_LOG2) {
                            need = true;
                            fac = fast_exp2(m_run - cms);
                            m_run = cms;
                            l_run *= fac;
                        }
                        if (__any_sync(0xffffffffu, need)) {   // scale this warp's O rows (previous PV done)
                            mbar_wait(&pv_done[(k - 1) & 1], ((k - 1) >> 1) & 1);
                            tc_fence_after();
                            for (int h = 0; h < d / 32; ++h) {
                                uint32_t ov[32];
                                tmem_ld32(tbase + lane_off + racc + 32 * h, ov);
                                tmem_wait_ld();
#pragma unroll
                                for (int e = 0; e < 32; ++e) ov[e] = __float_as_uint(__uint_as_float(ov[e]) * fac);
                                tmem_st16(tbase + lane_off + racc + 32 * h, *reinterpret_cast<const uint32_t(*)[16]>(&ov[0]));
                                tmem_st16(tbase + lane_off + racc + 32 * h + 16, *reinterpret_cast<const uint32_t(*)[16]>(&ov[16]));
                            }
                        }
                        float sum2[2] = {0.f, 0.f};
                        for (int c = 0; c < nch; ++c) {
                            if (c < clo || c > chi) {
                                tmem_st16(rS + c * 32, zero16);
                                tmem_st16(rS + c * 32 + 16, zero16);
                                continue;
                            }
#pragma unroll
                            for (int hh = 0; hh < 2; ++hh) {
                                const int n0 = c * 32 + 16 * hh;
                                uint32_t rr[16], pk[8], pl[8];
                                tmem_ld16(rS + n0, rr);
                                tmem_wait_ld();
#pragma unroll
                                for (int e = 0; e < 16; e += 2) {
                                    float a0, a1;
                                    ffma2_bc(__uint_as_float(rr[e]), __uint_as_float(rr[e + 1]), LOG2E, -m_run, a0, a1);
                                    const int n = n0 + e;
                                    const float p0 = (unsigned)(n - t + sh) <= (unsigned)W2 && kb + n >= 0 && kb + n < Lr ? fast_exp2(a0) : 0.f;
                                    const float p1 = (unsigned)(n + 1 - t + sh) <= (unsigned)W2 && kb + n + 1 >= 0 && kb + n + 1 < Lr ? fast_exp2(a1) : 0.f;
                                    fadd2_acc(sum2[0], sum2[1], p0, p1);
                                    split2(p0, p1, pk[e / 2], pl[e / 2]);
                                }
                                tmem_st8(rS + n0, pk);
                                tmem_st8(rS + n0 + 8, pl);
                            }
                        }
                        l_run += sum2[0] + sum2[1];
                        tmem_wait_st();
                        tc_fence_before();
                        warp_arrive(&p_full[k & 1]);
                        if (sb == nsb - 1) {   // 1/l and lse of the tile (the epilogue waits rs_full)
                            rowScale[(j % 3) * 128 + t] = 1.f / l_run;
                            if (rowv) p.lse[rowbase + (int64_t)mrow * p.dil] = (m_run + log2f(l_run)) * LN2;
                            warp_arrive(&rs_full[j & 1]);
                        }
                    } else if (MODE == BWDQ) {   // dS = P (dP - D) -> hi | lo over S
                        for (int c = 0; c < nch; ++c) {
                            if (!mine(c)) continue;
                            if (c < clo || c > chi) {
                                tmem_st16(rS + c * 32, zero16);
                                tmem_st16(rS + c * 32 + 16, zero16);
                                continue;
                            }
#pragma unroll
                            for (int hh = 0; hh < 2; ++hh) {
                                const int n0 = c * 32 + 16 * hh;
                                uint32_t rs[16], rd[16], pk[8], pl[8];
                                tmem_ld16(rS + n0, rs);
                                tmem_ld16(rP + n0, rd);
                                tmem_wait_ld();
#pragma unroll
                                for (int e = 0; e < 16; e += 2) {
                                    float a0, a1, q0, q1, d0, d1;
                                    const int n = n0 + e;
                                    ffma2_bc(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, -lse2, a0, a1);
                                    const float p0 = (unsigned)(n - t + sh) <= (unsigned)W2 && kb + n >= 0 && kb + n < Lr ? fast_exp2(a0) : 0.f;
                                    const float p1 = (unsigned)(n + 1 - t + sh) <= (unsigned)W2 && kb + n + 1 >= 0 && kb + n + 1 < Lr ? fast_exp2(a1) : 0.f;
                                    ffma2_bc(__uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), 1.f, -Drow, q0, q1);
                                    fmul2(p0, p1, q0, q1, d0, d1);
                                    split2(d0, d1, pk[e / 2], pl[e / 2]);
                                }
                                tmem_st8(rS + n0, pk);
                                tmem_st8(rS + n0 + 8, pl);
                            }
                        }
                        tmem_wait_st();
                        tc_fence_before();
                        warp_arrive(&p_full[k & 1]);
                    } else {   // BWDKV: rows keys, columns halo queries; P^T over dP^T, dS^T over S^T
                        for (int c = 0; c < nch; ++c) {
                            if (!mine(c)) continue;
                            if (c < clo || c > chi) {
                                tmem_st16(rS + c * 32, zero16);
                                tmem_st16(rS + c * 32 + 16, zero16);
                                tmem_st16(rP + c * 32, zero16);
                                tmem_st16(rP + c * 32 + 16, zero16);
                                continue;
                            }
#pragma unroll
                            for (int hh = 0; hh < 2; ++hh) {
                                const int n0 = c * 32 + 16 * hh;
                                uint32_t rs[16], rd[16], pk[8], pl[8], dk[8], dl[8];
                                tmem_ld16(rS + n0, rs);
                                tmem_ld16(rP + n0, rd);
                                tmem_wait_ld();
#pragma unroll
                                for (int e = 0; e < 16; e += 2) {
                                    float pv[2], dv[2], a0, a1, q0, q1;
                                    const int n = n0 + e;
                                    ffma2(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, LOG2E, -colLse[n], -colLse[n + 1], a0, a1);
                                    pv[0] = (unsigned)(n - t + sh) <= (unsigned)W2 && kb + n >= 0 && kb + n < Lr ? fast_exp2(a0) : 0.f;
                                    pv[1] = (unsigned)(n + 1 - t + sh) <= (unsigned)W2 && kb + n + 1 >= 0 && kb + n + 1 < Lr ? fast_exp2(a1) : 0.f;
                                    ffma2(__uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), 1.f, 1.f, -colD[n], -colD[n + 1], q0, q1);
                                    fmul2(pv[0], pv[1], q0, q1, dv[0], dv[1]);
                                    split2(pv[0], pv[1], pk[e / 2], pl[e / 2]);
                                    split2(dv[0], dv[1], dk[e / 2], dl[e / 2]);
                                }
                                tmem_st8(rS + n0, dk);          // dS^T over S^T
                                tmem_st8(rS + n0 + 8, dl);
                                tmem_st8(rP + n0, pk);          // P^T over dP^T
                                tmem_st8(rP + n0 + 8, pl);
                            }
                        }
                        tmem_wait_st();
                        tc_fence_before();
                        warp_arrive(&p_full[k & 1]);
                    }
                }
                if (SPLITSM && hsm == 1) drain_tile(T, j, sidx, euses, 1.f);
                ++j;
            }
            if (SPLITSM && hsm == 1 && lane == 0) tma_store_wait_all<0>();
        }
        bool lse_settled = false;   // ld_lse_ready fell back to griddepcontrol.wait
        while (!WIDE && cur.next(p.sc, T)) {
            const int Lr = T.Lr, m0 = T.m0, mrow = m0 + t, kb = m0 - w;
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            if (MODE == BWDKV && !XT) {
                named_bar_sync(1, 128);   // everyone is done with the previous tile's columns
                for (int n = t; n < NK; n += 128) {
                    const int mc = kb + n;
                    const bool ok = mc >= 0 && mc < Lr;
                    colLse[n] = !ok ? 0.f
                                : (p.lsepoll ? ld_lse_ready(p.lse + rowbase + (int64_t)mc * p.dil, lse_settled)
                                             : p.lse[rowbase + (int64_t)mc * p.dil]) * LOG2E;
                    float dv = 0.f;
                    if (ok) dv = p.dpoll ? ld_D_ready(p.D + rowbase + (int64_t)mc * p.dil) : p.D[rowbase + (int64_t)mc * p.dil];
                    colD[n] = dv;
                }
                named_bar_sync(1, 128);
            }
            const int sidx = MODE == FWD ? (j & 1) : 0;
            const uint32_t sph = MODE == FWD ? ((j >> 1) & 1) : (j & 1);
            if (!xt) {
                mbar_wait(&s_full[sidx], sph);
                tc_fence_after();
            }
            if (t == 0) trace_tile(p, j, 0);
            const uint32_t rS = tbase + lane_off + (MODE == FWD && (j & 1) ? R1 : R0);
            const uint32_t rP = tbase + lane_off + R1;
            // The bf16 operand of 16 keys (K-step g = key / 16) is packed in place over those keys'
            // 16 fp32 columns: hi words at columns [16 g, 16 g + 8), lo words at [16 g + 8, 16 g + 16).
            if (MODE == FWD) {
                float mx = -INFINITY;
                for (int c = c_lo; c <= c_hi; ++c) {
                    uint32_t rr[32];
                    tmem_ld32(rS + c * 32, rr);
                    tmem_wait_ld();
#pragma unroll
                    for (int e = 0; e < 32; ++e)
                        if (band_ok(c * 32 + e, t, w, kb + c * 32 + e, Lr)) mx = fmaxf(mx, __uint_as_float(rr[e]));
                }
                if (mx == -INFINITY) mx = 0.f;   // rows beyond the sequence (never stored)
                const float mxs = mx * LOG2E;
                float sum2[2] = {0.f, 0.f};
                for (int c = 0; c < nch; ++c) {
                    if (c < c_lo || c > c_hi) {
                        tmem_st16(rS + c * 32, zero16);
                        tmem_st16(rS + c * 32 + 16, zero16);
                        continue;
                    }
#pragma unroll
                    for (int hh = 0; hh < 2; ++hh) {
                        const int n0 = c * 32 + 16 * hh;
                        uint32_t rr[16], pk[8], pl[8];
                        tmem_ld16(rS + n0, rr);
                        tmem_wait_ld();
#pragma unroll
                        for (int e = 0; e < 16; e += 2) {   // packed f32x2 pairs, two partial sums
                            float a0, a1;
                            ffma2_bc(__uint_as_float(rr[e]), __uint_as_float(rr[e + 1]), LOG2E, -mxs, a0, a1);
                            const int n = n0 + e;
                            const float p0 = band_ok(n, t, w, kb + n, Lr) ? fast_exp2(a0) : 0.f;
                            const float p1 = band_ok(n + 1, t, w, kb + n + 1, Lr) ? fast_exp2(a1) : 0.f;
                            fadd2_acc(sum2[0], sum2[1], p0, p1);
                            split2(p0, p1, pk[e / 2], pl[e / 2]);
                        }
                        tmem_st8(rS + n0, pk);
                        tmem_st8(rS + n0 + 8, pl);
                    }
                }
                const float sum = sum2[0] + sum2[1];
                rowScale[(j % 3) * 128 + t] = 1.f / sum;
                tmem_wait_st();
                tc_fence_before();
                warp_arrive(&p_full[j & 1]);
                if (t == 0) trace_tile(p, j, 1);
                if (mrow < Lr) p.lse[rowbase + (int64_t)mrow * p.dil] = (mxs + log2f(sum)) * LN2;
            } else if (MODE == BWDQ) {
                const float lse2 = mrow >= Lr ? 0.f
                                   : (p.lsepoll ? ld_lse_ready(p.lse + rowbase + (int64_t)mrow * p.dil, lse_settled)
                                                : p.lse[rowbase + (int64_t)mrow * p.dil]) * LOG2E;
                float Dp[4] = {0.f, 0.f, 0.f, 0.f};   // four partial sums (FFMA2 pairs)
                for (int c = c_lo; c <= c_hi; ++c) {   // pass 1: D = sum_j P_ij dP_ij
#pragma unroll
                    for (int hh = 0; hh < 2; ++hh) {
                        const int n0 = c * 32 + 16 * hh;
                        uint32_t rs[16], rd[16];
                        tmem_ld16(rS + n0, rs);
                        tmem_ld16(rP + n0, rd);
                        tmem_wait_ld();
#pragma unroll
                        for (int e = 0; e < 16; e += 2) {
                            float a0, a1;
                            ffma2_bc(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, -lse2, a0, a1);
                            const int n = n0 + e, q = e & 2;
                            const float p0 = band_ok(n, t, w, kb + n, Lr) ? fast_exp2(a0) : 0.f;
                            const float p1 = band_ok(n + 1, t, w, kb + n + 1, Lr) ? fast_exp2(a1) : 0.f;
                            ffma2(p0, p1, __uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), Dp[q], Dp[q + 1], Dp[q], Dp[q + 1]);
                        }
                    }
                }
                const float D = (Dp[0] + Dp[1]) + (Dp[2] + Dp[3]);
                for (int c = 0; c < nch; ++c) {   // pass 2: dS = P (dP - D) -> hi | lo over S
                    if (c < c_lo || c > c_hi) {
                        tmem_st16(rS + c * 32, zero16);
                        tmem_st16(rS + c * 32 + 16, zero16);
                        continue;
                    }
#pragma unroll
                    for (int hh = 0; hh < 2; ++hh) {
                        const int n0 = c * 32 + 16 * hh;
                        uint32_t rs[16], rd[16], pk[8], pl[8];
                        tmem_ld16(rS + n0, rs);
                        tmem_ld16(rP + n0, rd);
                        tmem_wait_ld();
                        // tape entry e = n - t of row mrow sits at float (mrow & 3) + e = ob + (n - n0):
                        // four entries per 16-byte store ((mrow & 3) == (t & 3), m0 % 128 == 0)
                        const int ob = (t & 3) + n0 - t;
#pragma unroll
                        for (int g4 = 0; g4 < 4; ++g4) {
                            float pv[4], dv[4];
#pragma unroll
                            for (int x = 0; x < 4; x += 2) {   // packed f32x2 pairs
                                const int n = n0 + 4 * g4 + x, i = 4 * g4 + x;
                                float a0, a1, q0, q1;
                                ffma2_bc(__uint_as_float(rs[i]), __uint_as_float(rs[i + 1]), LOG2E, -lse2, a0, a1);
                                pv[x] = band_ok(n, t, w, kb + n, Lr) ? fast_exp2(a0) : 0.f;
                                pv[x + 1] = band_ok(n + 1, t, w, kb + n + 1, Lr) ? fast_exp2(a1) : 0.f;
                                ffma2_bc(__uint_as_float(rd[i]), __uint_as_float(rd[i + 1]), 1.f, -D, q0, q1);
                                fmul2(pv[x], pv[x + 1], q0, q1, dv[x], dv[x + 1]);
                            }
                            split2(dv[0], dv[1], pk[2 * g4], pl[2 * g4]);
                            split2(dv[2], dv[3], pk[2 * g4 + 1], pl[2 * g4 + 1]);
                            const int o = ob + 4 * g4;
                            if (XT && mrow < Lr && o >= 0 && o < p.tsw) {
                                const size_t ro = ((size_t)(o >> 2) * p.grows + rowbase + (int64_t)mrow * p.dil) * 4;
                                *reinterpret_cast<float4*>(p.tP + ro) = make_float4(pv[0], pv[1], pv[2], pv[3]);
                                *reinterpret_cast<float4*>(p.tS + ro) = make_float4(dv[0], dv[1], dv[2], dv[3]);
                            }
                        }
                        tmem_st8(rS + n0, pk);
                        tmem_st8(rS + n0 + 8, pl);
                    }
                }
                tmem_wait_st();
                tc_fence_before();
                warp_arrive(&p_full[j & 1]);
                if (mrow < Lr) p.D[rowbase + (int64_t)mrow * p.dil] = D;
                if (XT) {   // publish the tile's tape rows to BWDKV
                    __threadfence();
                    named_bar_sync(2, 128);
                    if (t == 0) st_release_gpu(p.flags + rowbase + (int64_t)m0 * p.dil, 1u);
                }
            } else if (xt) {   // BWDKV from the dS tape: P^T -> R1 (hi | lo), then dS^T -> R0

                // walk positions (see walk): every segment holds 2 ncw nkb output blocks and 2 npl tape slots, plus P(0) in
                // segment 0; P(j > 0) is the npl slots before the last dK chunk of segment j - 1
                const int seg = nacc * nkb + 2 * npl;
                const int Sj = j * seg + (j > 0 ? npl : 0);
                const int posP = j == 0 ? 0 : Sj - nkb - npl;
                const int posS = Sj + (j == 0 ? npl : 0) + (ncw - 1) * nkb;
                for (int h = 0; h < 2; ++h) {
                    // R1 once the previous tile's dK accumulations in it are drained; R0 once this
                    // tile's dV accumulations in it are (the MMAs that read them as A came earlier)
                    if (h == 1) mbar_wait(&xfree[1], (uint32_t)j & 1u);
                    else if (j > 0) mbar_wait(&xfree[0], (uint32_t)(j - 1) & 1u);
                    tc_fence_after();
                    if (t == 0) trace_tile(p, j, 10 + 3 * h);   // operand region free
                    const uint32_t dst = h == 0 ? rP : rS;
                    for (int b = 0; b < npl; ++b) {
                        const int k = (h ? posS : posP) + b, st = k % nst;
                        mbar_wait(&full[st], (uint32_t)(k / nst) & 1u);
                        if (t == 0 && b == 0) trace_tile(p, j, 11 + 3 * h);   // first tape slot landed
                        const float* sv = reinterpret_cast<const float*>(slots + (size_t)st * slotb);
                        for (int c = 3 * b; c < 3 * b + 3 && c < nch; ++c) {
                            if (c < c_lo || c > c_hi) {
                                tmem_st16(dst + c * 32, zero16);
                                tmem_st16(dst + c * 32 + 16, zero16);
                                continue;
                            }
#pragma unroll
                            for (int hh = 0; hh < 2; ++hh) {
                                // column n = n0 + e (query kb + n, tape row n - 96 b of the slot), key
                                // t: offset o = (kb + n) & 3 + t - n + 2w, at float (o / 4) 4 TBOX +
                                // (n - 96 b) 4 + o % 4 of the slot; in the band iff e in [lo, hi].
                                // Branch-free, loads back to back.
                                const int n0 = c * 32 + 16 * hh;
                                const int lo = max(t - n0, -(kb + n0)), hi = min(t - n0 + 2 * w, Lr - 1 - (kb + n0));
                                uint32_t pk[8], pl[8];
                                float x[16];
#pragma unroll
                                for (int e = 0; e < 16; ++e) {
                                    const int n = n0 + e;
                                    const int o = ((kb + n) & 3) + t - n + 2 * w;
                                    const bool ok = e >= lo && e <= hi;
                                    const float xv = sv[ok ? (o >> 2) * (4 * TBOX) + (n - TROWS * b) * 4 + (o & 3) : 0];
                                    x[e] = ok ? xv : 0.f;
                                }
#pragma unroll
                                for (int e = 0; e < 16; e += 2) split2(x[e], x[e + 1], pk[e / 2], pl[e / 2]);
                                tmem_st8(dst + n0, pk);
                                tmem_st8(dst + n0 + 8, pl);
                            }
                        }
                        named_bar_sync(1, 128);   // all four warps are done with this slot
                        if (t == 0) mbar_arrive(&empty[st]);
                    }
                    tmem_wait_st();
                    tc_fence_before();
                    warp_arrive(&p_full[h]);
                    if (t == 0) trace_tile(p, j, 12 + 3 * h);   // operand built
                }
            } else {   // BWDKV: rows are keys, columns halo queries
                for (int c = 0; c < nch; ++c) {
                    if (c < c_lo || c > c_hi) {
                        tmem_st16(rS + c * 32, zero16);
                        tmem_st16(rS + c * 32 + 16, zero16);
                        tmem_st16(rP + c * 32, zero16);
                        tmem_st16(rP + c * 32 + 16, zero16);
                        continue;
                    }
#pragma unroll
                    for (int hh = 0; hh < 2; ++hh) {
                        const int n0 = c * 32 + 16 * hh;
                        uint32_t rs[16], rd[16], pk[8], pl[8], dk[8], dl[8];
                        tmem_ld16(rS + n0, rs);
                        tmem_ld16(rP + n0, rd);
                        tmem_wait_ld();
#pragma unroll
                        for (int e = 0; e < 16; e += 2) {
                            float pv[2], dv[2], a0, a1, q0, q1;   // packed f32x2 pairs
                            const int n = n0 + e;
                            ffma2(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, LOG2E, -colLse[n], -colLse[n + 1], a0, a1);
                            pv[0] = band_ok(n, t, w, kb + n, Lr) ? fast_exp2(a0) : 0.f;
                            pv[1] = band_ok(n + 1, t, w, kb + n + 1, Lr) ? fast_exp2(a1) : 0.f;
                            ffma2(__uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), 1.f, 1.f, -colD[n], -colD[n + 1], q0, q1);
                            fmul2(pv[0], pv[1], q0, q1, dv[0], dv[1]);
                            split2(pv[0], pv[1], pk[e / 2], pl[e / 2]);
                            split2(dv[0], dv[1], dk[e / 2], dl[e / 2]);
                        }
                        tmem_st8(rS + n0, dk);          // dS^T over S^T
                        tmem_st8(rS + n0 + 8, dl);
                        tmem_st8(rP + n0, pk);          // P^T over dP^T
                        tmem_st8(rP + n0 + 8, pl);
                    }
                }
                tmem_wait_st();
                tc_fence_before();
                warp_arrive(&p_full[j & 1]);
            }
            ++j;
        }
    } else if (warp < 8) {   // ----------------------------------------------- epilogue warps
        TileCursor cur(p.sc);
        Tile T;
        int j = 0, sidx = 0;
        AccUses uses;
        while (cur.next(p.sc, T)) {
            float scale = 1.f;
            if (MODE == FWD) {   // 1/l of this row, published before p_full (WIDE: rs_full)
                if (WIDE) mbar_wait(&rs_full[j & 1], (j >> 1) & 1);
                else mbar_wait(&p_full[j & 1], (j >> 1) & 1);
                scale = rowScale[(j % 3) * 128 + (warp - 4) * 32 + lane];
            }
            drain_tile(T, j, sidx, uses, scale);
            ++j;
        }
        if (lane == 0) tma_store_wait_all<0>();
    }
    tc_fence_before();
    // (a PDL-launched grid that never waited must not complete before its primary: stream order
    // for whatever follows it)
    if (p.pdl_free) asm volatile("griddepcontrol.wait;" ::: "memory");
    __syncthreads();
    if (warp == 8) {
        tc_fence_after();
        tmem_dealloc(tbase, 512);
    }
}

int num_sms32() {
    static int n = 0;
    static std::once_flag once;
    std::call_once(once, [] {
        int dev = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0)
            n = 148;
    });
    return n;
}

int halo_rows32(int64_t L, int64_t w) {
    const int64_t wc = w < L ? w : L;
    return (int)(((BM + 2 * wc) + 63) / 64 * 64);
}

// WIDE steps: ceil((128 + 2w) / NK) halo windows of NK rows per tile (NK = 192 at d = 64, 128 at
// d = 128; w clamped to the longest residue), at most WMAX_SB.
// The steps are balanced: n = ceil(halo / NKmax) steps (NKmax = 192 at d = 64, 128 at d = 128) of
// NK = halo / n rows rounded up to 32 -- e.g. 4 x 160 for w = 256 instead of 3 x 192 + a 64-row
// remainder that costs a whole step.  At d = 64 with NK <= 160 a step's keys form one output
// block (NK x 64 fp32 <= one 40 KB slot); otherwise blocks of KB = 64 keys (NK a multiple of 64).
struct WideGeo {
    int n, nk, kbw;
};
inline bool wide_geo(int64_t L, int64_t w, int64_t dil, int64_t d, WideGeo& g) {
    const int64_t Lr = (L + dil - 1) / dil;
    const int64_t wm = w < Lr ? w : Lr;
    const int64_t halo = BM + 2 * wm, nkmax = d == 128 ? 128 : 192;
    const int64_t n = (halo + nkmax - 1) / nkmax;
    if (n > WMAX_SB) return false;
    int64_t nk = ((halo + n - 1) / n + 31) / 32 * 32;
    int kbw = (int)nk;
    if (!(d == 64 && nk <= 160)) {
        nk = (nk + 63) / 64 * 64;
        kbw = KB;
    }
    if (nk > nkmax) return false;
    g.n = (int)n;
    g.nk = (int)nk;
    g.kbw = kbw;
    return true;
}

// D_i = dout_i . out_i (fp32; the WIDE backward's exact-to-rounding D, reading R1 for fp32 out):
// one warp per row, d a multiple of 64.
__global__ void __launch_bounds__(256) rowdot32_kernel(const float* __restrict__ out, const float* __restrict__ dout,
                                                       float* __restrict__ D, int64_t rows, int d) {
    const int64_t r = (int64_t)blockIdx.x * 8 + threadIdx.x / 32;
    const int lane = threadIdx.x % 32;
    if (r >= rows) return;
    const float* o = out + r * d;
    const float* g = dout + r * d;
    float acc = 0.f;
    for (int c = 2 * lane; c < d; c += 64) {
        const float2 a = __ldg(reinterpret_cast<const float2*>(o + c));
        const float2 b = __ldg(reinterpret_cast<const float2*>(g + c));
        acc = fmaf(a.x, b.x, fmaf(a.y, b.y, acc));
    }
#pragma unroll
    for (int x = 16; x >= 1; x >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, x);
    if (lane == 0) D[r] = acc;
}

template <int MODE, bool WIDE>
cudaError_t launch32(const void* a1, const void* b1, const void* a2, const void* b2, const void* ob1,
                     const void* ob2, void* o1, void* o2, float* lse, float* D, const DsTape* tape, int64_t B,
                     int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st, int* launches) {
    constexpr bool HAS_XT = MODE != FWD && !WIDE;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_band32_kernel<MODE, WIDE, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)SMEM_BYTES);
        if constexpr (HAS_XT)
            cudaFuncSetAttribute(tc_band32_kernel<MODE, WIDE, HAS_XT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)(SMEM_BYTES > SMEM_BYTES_XT ? SMEM_BYTES : SMEM_BYTES_XT));
    });
    const int64_t wc = w < L ? w : L;
    WideGeo wg = {1, 0, KB};
    if (WIDE && !wide_geo(L, w, dil, d, wg)) return cudaErrorInvalidValue;
    const int NK = WIDE ? wg.nk : halo_rows32(L, w);
    const int nsteps = WIDE ? wg.n : 1;
    const int kbw = WIDE ? wg.kbw : KB;
    if (WIDE) tape = nullptr;
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        Params p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            Maps& m = p.maps[i];
            bool ok = make_residue_map_f32(&m.a1, a1, L, d, units, dil, r, BM, 16) &&
                      make_residue_map_f32(&m.b1, b1, L, d, units, dil, r, NK, 16) &&
                      make_residue_map_f32(&m.ob1, ob1, L, d, units, dil, r, kbw) &&
                      make_residue_map_f32(&m.o1, o1, L, d, units, dil, r, 32);
            if (ok && a2) ok = make_residue_map_f32(&m.a2, a2, L, d, units, dil, r, BM, 16);
            if (ok && b2) ok = make_residue_map_f32(&m.b2, b2, L, d, units, dil, r, NK, 16);
            if (ok && ob2) ok = make_residue_map_f32(&m.ob2, ob2, L, d, units, dil, r, kbw);
            if (ok && o2) ok = make_residue_map_f32(&m.o2, o2, L, d, units, dil, r, 32);
            if (ok && tape && MODE == BWDKV && d > CW) {
                ok = make_residue_map_tape(&m.tp, tape->P, L, tape->tsw, units, dil, r, TBOX, tape->grows) &&
                     make_residue_map_tape(&m.ts, tape->S, L, tape->tsw, units, dil, r, TBOX, tape->grows);
            }
            if (!ok) return cudaErrorInvalidValue;
        }
        p.lse = lse;
        p.D = D;
        p.L = L;
        p.d = (int)d;
        p.w = WIDE ? (int)(wc < ceil_div(L, dil) ? wc : ceil_div(L, dil)) : (int)wc;   // (wide_steps' clamp)
        p.dil = (int)dil;
        p.NK = NK;
        p.nsl = (int)(d / 32);
        p.dpoll = MODE != FWD && dpoll_enabled() && !WIDE;   // BWDQ marks its D rows, BWDKV polls them
        if (WIDE) p.nsb = nsteps;
        p.kbw = kbw;
        // WIDE: the dK/dV kernel needs only lse and D (both final before the dQ kernel starts), so it
        // runs beside the dQ kernel as SMs free up
        p.pdl_free = WIDE && MODE == BWDKV && r0 == 0 && dpoll_enabled();
        if (tape && MODE != FWD && d > CW) {   // xt needs two output chunks (acc_rid alternation)
            p.xt = 1;
            p.tsw = tape->tsw;
            p.grows = tape->grows;
            p.flags = tape->flags;
            p.tP = tape->P;
            p.tS = tape->S;
        }
        p.trace = (unsigned long long*)trace_buffer(MODE);
        const int64_t Lr0 = ceil_div(L - r0, dil);
        const int tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = units * nr * tiles;
        dim3 grid((unsigned)(total < num_sms32() ? total : num_sms32()));
        const size_t smem = MODE == BWDKV && p.xt ? SMEM_BYTES_XT : SMEM_BYTES;
        void (*kern)(Params) = tc_band32_kernel<MODE, WIDE, false>;
        if constexpr (HAS_XT)
            if (p.xt) kern = tc_band32_kernel<MODE, WIDE, HAS_XT>;
        sched_init(p.sc, L, dil, r0, nr, units, tiles, (int)grid.x);
        // lse hand-off: one launch of residues on each side (nres <= RES_PER_LAUNCH) -- the
        // dQ kernel's launch follows the forward's only launch
        p.lsepoll = lsepoll_enabled() && nres <= RES_PER_LAUNCH && lsepoll_worth(total, num_sms32()) &&
                    !(MODE == BWDKV && p.xt) && !WIDE;   // the tape dK/dV kernel reads no lse
        if ((MODE == BWDKV && r0 == 0 && p.dpoll) || (MODE == BWDQ && p.lsepoll) || p.pdl_free) {
            // BWDKV directly after this call's last BWDQ launch; BWDQ after the forward
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = grid;
            cfg.blockDim = dim3(NTHREADS);
            cfg.dynamicSmemBytes = smem;
            cfg.stream = st;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            at[0].val.programmaticStreamSerializationAllowed = 1;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            cudaLaunchKernelEx(&cfg, kern, p);
        } else {
            kern<<<grid, NTHREADS, smem, st>>>(p);
        }
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        ++n;
    }
    if (launches) *launches += n;
    return cudaSuccess;
}

int band32_launches(int64_t L, int64_t dil) {
    const int64_t nres = dil < L ? dil : L;
    return (int)ceil_div(nres, RES_PER_LAUNCH);
}

}  // namespace

// w > 32 runs the WIDE instantiation: d = 64 (192-row steps; dV and dK share the 128 accumulator
// columns) or d = 128 (128-row steps; dV and dK take 128 columns each)
static bool tc32_wide(int64_t L, int64_t w) { return (w < L ? w : L) > 32; }
bool tc32_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    const int64_t wc = w < L ? w : L;
    if (!(dil <= 256 && units * ((L + 127) / 128) < (1 << 30))) return false;
    if (wc <= 32) return d % 64 == 0 && d <= 512;
    WideGeo g;
    return (d == 64 || d == 128) && wide_geo(L, w, dil, d, g);
}
int tc32_fwd_launches(int64_t L, int64_t w, int64_t dil) { return band32_launches(L, dil); }
int tc32_bwd_launches(int64_t L, int64_t w, int64_t dil) { return 2 * band32_launches(L, dil) + (tc32_wide(L, w) ? 1 : 0); }

cudaError_t tc32_fwd(const void* q, const void* k, const void* v, void* out, float* lse, int64_t B, int64_t H,
                     int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st, int* launches) {
    if (launches) *launches = 0;
    if (tc32_wide(L, w))
        return launch32<FWD, true>(q, k, nullptr, nullptr, v, nullptr, out, nullptr, lse, nullptr, nullptr, B, H, L,
                                   d, w, dil, st, launches);
    return launch32<FWD, false>(q, k, nullptr, nullptr, v, nullptr, out, nullptr, lse, nullptr, nullptr, B, H, L, d, w,
                                dil, st, launches);
}

cudaError_t tc32_bwd(const void* q, const void* k, const void* v, const void* out, const float* lse, const void* dout,
                     void* dq, void* dk, void* dv, float* Dws, const DsTape* tape, int64_t B, int64_t H, int64_t L,
                     int64_t d, int64_t w, int64_t dil, cudaStream_t st, int* launches) {
    if (launches) *launches = 0;
    if (tc32_wide(L, w)) {   // D = dout . out first; then the two kernels, independent of each other
        const int64_t rows = B * H * L;
        rowdot32_kernel<<<(unsigned)((rows + 7) / 8), 256, 0, st>>>((const float*)out, (const float*)dout, Dws, rows, (int)d);
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        if (launches) *launches += 1;
        e = launch32<BWDQ, true>(q, k, dout, v, k, nullptr, dq, nullptr, const_cast<float*>(lse), Dws, nullptr, B, H,
                                 L, d, w, dil, st, launches);
        if (e != cudaSuccess) return e;
        return launch32<BWDKV, true>(k, q, v, dout, dout, q, dk, dv, const_cast<float*>(lse), Dws, nullptr, B, H, L, d,
                                     w, dil, st, launches);
    }
    // BWDQ: S = Q K_h^T (a1 = q, b1 = k), dP = dO V_h^T (a2 = dout, b2 = v), dQ = dS K_h (ob1 = k)
    cudaError_t e = launch32<BWDQ, false>(q, k, dout, v, k, nullptr, dq, nullptr, const_cast<float*>(lse), Dws, tape,
                                          B, H, L, d, w, dil, st, launches);
    if (e != cudaSuccess) return e;
    // BWDKV: S^T = K Q_h^T, dP^T = V dO_h^T; dV = P^T dO_h (ob1 = dout -> o2 = dv), dK = dS^T Q_h
    // (ob2 = q -> o1 = dk).  Accumulations: dV chunks (a < ncw, o2), then dK chunks (o1).
    // With the dS tape (PAPER.md:489-497 selective materialization) BWDKV skips S^T and dP^T: it
    // streams only the tape rows and the dO / Q blocks of its output GEMMs.
    return launch32<BWDKV, false>(k, q, v, dout, dout, q, dk, dv, const_cast<float*>(lse), Dws, tape, B, H, L, d, w,
                                  dil, st, launches);
}

}  // namespace ftw
