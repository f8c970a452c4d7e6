// tile_sched.cuh -- division-free static round-robin tile cursor for the persistent kernels.
//
// Tile tau = (unit * nr + rl) * tiles + t  (row block t fastest, so concurrently running
// CTAs work on neighbouring row blocks and share their halos through L2).  A CTA visits
// tau = blockIdx.x, blockIdx.x + G, ... (G = gridDim.x).  Decoding tau with divisions costs a
// long dependent chain (~1000 cycles with the int64 residue length), which sat on every role's
// critical path between tiles (tools/trace_narrow.py); the cursor below advances (t, rl, u)
// by G with precomputed quotients and one carry each, and tests the tile against the residue
// length table filled on the host.
#pragma once
#include <stdint.h>

namespace ftw {

constexpr int SCHED_MAX_RES = 8;   // >= every kernel's residues per launch (static_asserts)

struct SchedParams {
    int tiles;                 // row blocks per residue (of the longest residue of the launch)
    int nr;                    // residues in this launch
    int units;                 // batch * heads
    int r0;                    // first residue of this launch
    int dt, dres_mod, dres_div;   // G % tiles, (G / tiles) % nr, (G / tiles) / nr
    int Lr[SCHED_MAX_RES];     // rows of each residue: ceil((L - r) / dilation)
};

inline void sched_init(SchedParams& s, int64_t L, int64_t dil, int64_t r0, int nr, int64_t units,
                       int tiles, int grid) {
    s.tiles = tiles;
    s.nr = nr;
    s.units = (int)units;
    s.r0 = (int)r0;
    s.dt = grid % tiles;
    const int dres = grid / tiles;
    s.dres_mod = dres % nr;
    s.dres_div = dres / nr;
    for (int i = 0; i < SCHED_MAX_RES; ++i)
        s.Lr[i] = i < nr ? (int)((L - (r0 + i) + dil - 1) / dil) : 0;
}

struct SchedTile {
    int u, rl, r, Lr, m0;
};

template <int BM>
struct SchedCursor {
    int t, rl, u;
    bool started;
    __device__ explicit SchedCursor(const SchedParams& s) : started(false) {
        const int tau = blockIdx.x;   // one-time divisions
        t = tau % s.tiles;
        const int rest = tau / s.tiles;
        rl = rest % s.nr;
        u = rest / s.nr;
    }
    __device__ __forceinline__ void step(const SchedParams& s) {
        t += s.dt;
        int c = 0;
        if (t >= s.tiles) { t -= s.tiles; c = 1; }
        rl += s.dres_mod + c;
        u += s.dres_div;
        if (rl >= s.nr) { rl -= s.nr; u += 1; }
    }
    // next valid tile of this CTA; false when the CTA is done
    __device__ __forceinline__ bool next(const SchedParams& s, SchedTile& T) {
        if (started) step(s);
        started = true;
        for (; u < s.units; step(s)) {
            const int Lr = s.Lr[rl];
            if (t * BM < Lr) {
                T.u = u;
                T.rl = rl;
                T.r = s.r0 + rl;
                T.Lr = Lr;
                T.m0 = t * BM;
                return true;
            }
        }
        return false;
    }
};

}  // namespace ftw
