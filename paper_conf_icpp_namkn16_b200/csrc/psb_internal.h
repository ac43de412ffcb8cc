// psb_internal.h — definitions shared by the host builder, the C ABI and the
// CUDA kernels of libpsb.so (never by the oracle).
#pragma once
#include <stdint.h>

#include "psb.h"

#define PSB_MAXLVL 8   // internal levels; F=32 and n < 2^31 need at most 6
// Large batches at d <= this are ordered by Hilbert key instead of closest leaf
// (knn_order.cu; DESIGN.md §6 "Batch scheduling").
#ifndef PSB_HILBERT_ORDER_MAX_D
#define PSB_HILBERT_ORDER_MAX_D 4
#endif

// Flat index as laid out in HBM (DESIGN.md §4 "Data layout in HBM").
//   pts   [L][d][F]  leaf-blocked SoA point coordinates (pad slots +inf)
//   ids   [L][F]     global point ids (pad slots -1)
//   nodes levels 1..H; level l holds nlev[l] blocks of [d][2][F] child MBRs
//         (row 2j = lo of dim j, row 2j+1 = hi of dim j; empty slot lo=+inf hi=-inf)
// Packed-tree closed forms: children of (l, i) are
// (l-1, i*F + c); parent of (l, i) is (l+1, i/F); the leaves under (l, i) are
// [i*span[l], min((i+1)*span[l], L)), span[l] = F^l; right sibling of leaf j is j+1.
struct DevIndex {
    const float *pts;
    const int32_t *ids;
    const float *nodes;
    const float *box;                   // bounding box of the real points [2][d] (lo, hi)
    int64_t level_off[PSB_MAXLVL + 1];  // float offset of level l's first block (l >= 1)
    int64_t nlev[PSB_MAXLVL + 1];       // nodes per level, nlev[0] = L
    int64_t span[PSB_MAXLVL + 1];       // leaves per full subtree at level l (clamped)
    int64_t n;                          // real points
    int64_t L;                          // leaves
    int32_t H;                          // internal levels; root = (H, 0)
    int32_t d;
    int32_t F;
    int32_t sm_count;                   // of the index's device (launch sizing)
    int32_t sphere;                     // 0: MBR node blocks [d][2][F]; 1: sphere blocks [d+1][F]
    int32_t blk_floats;                 // floats per internal node block
    int32_t irregular;                  // imported tree whose leaves are not all full (but the last):
                                        // the count-aware MAXDIST bound (R3) does not apply
    // per launch (k known): a child (lvl-1, c) of a level-lvl node holds >= k points
    // iff c <= kcnt_lim[lvl] (every subtree but the level's last holds >= F points)
    int32_t kcnt_lim[PSB_MAXLVL + 1];
};

// psb_knn_trace output: per query, its traversal steps in order (kernels with
// counting compiled in only). buf [q][cap] (nullable), len [q] (nullable).
struct TraceOut {
    int64_t *buf;
    int32_t *len;
    int cap;
};

// Level geometry of a packed tree (shared by the host and GPU loaders).
struct GpuLayoutShape {
    int64_t n = 0, L = 0;
    int32_t d = 0, F = 0, H = 0;
    int32_t sphere = 0, blk_floats = 0;
    int64_t nlev[PSB_MAXLVL + 1] = {};
    int64_t level_off[PSB_MAXLVL + 1] = {};
    int64_t total_node_floats = 0;
};

// Validates (n, d, F, id_base, flags) and computes the geometry; PSB_OK or an
// error code with the message set. Does not read the points.
int psb_layout_shape(int64_t n, int32_t d, int32_t F, int64_t id_base, uint32_t flags, GpuLayoutShape *s);

struct HostLayout {
    int64_t n = 0, L = 0, id_base = 0;
    int32_t d = 0, F = 0, H = 0;
    int64_t nlev[PSB_MAXLVL + 1] = {};
    int64_t level_off[PSB_MAXLVL + 1] = {};
    int64_t total_node_floats = 0;
    float *pts = nullptr;      // [L][d][F]
    int32_t *ids = nullptr;    // [L][F]
    float *nodes = nullptr;    // total_node_floats
    ~HostLayout();
};

// Host bulk loader (psb_build.cpp). Returns PSB_OK or an error code with the
// thread-local message set.
int psb_host_build(const float *points, int64_t n, int32_t d, int32_t F, int64_t id_base,
                   uint32_t flags, HostLayout *out);

void psb_set_error(const char *fmt, ...);
