// efg_kernels.cuh — launchers for the sm_100a kernels (efg_kernels.cu).
#pragma once

#include <cuda_runtime.h>

#include "efg_internal.h"

namespace efg {

enum ExpandMode : int {
    kModeVisit = 0,        // BFS: visited-bitmap probe + atomicOr (Alg. 1 lines 3-4)
    kModeVisitParent = 1,  // BFS with parents (winner of the atomicOr writes parent)
    kModeDecode = 2,       // efg_decode: store the decoded value in CSR order
};

struct ExpandArgs {
    const uint8_t *data;       // EF data (device, 4-byte aligned, padded)
    const VRec *rec;           // packed vertex records
    const uint32_t *queue;     // frontier queue
    const TileEntry *tiles;    // tile table
    const LevelCtrl *ctrl;     // nf, ne, ntiles of this level
    uint32_t *vis;             // visited bitmap (modes 0, 1)
    uint32_t *out;             // parent (mode 1) or decode output (mode 2)
    uint32_t k;                // forward-pointer quantum (chunk length); 0 = none
    int32_t kshift;            // log2(k) if k is a power of two, else -1
};

struct AdvanceArgs {
    uint32_t *vis;             // visited bitmap
    uint32_t *prev;            // visited bitmap after the previous advance
    const VRec *rec;
    const uint32_t *deg32;     // degrees (compact copy for the frontier step a1)
    int32_t *depth;            // depth output (may be the caller's device buffer)
    uint32_t *queue;           // next frontier (sorted by vertex id)
    TileEntry *tiles;          // tile table of the next level
    uint64_t *status;          // decoupled look-back status [2][2][nblocks]
    LevelCtrl *ctrl;           // totals of the next level
    uint64_t nwords;           // bitmap words
    uint64_t nblocks;          // grid size
    int32_t depth_value;       // depth assigned to newly discovered vertices
    uint32_t parity;           // status parity of this launch
    uint32_t k;                // chunk length (0 = whole lists)
    int32_t kshift;            // log2(k) if k is a power of two, else -1
};

cudaError_t launch_expand(int mode, const ExpandArgs &a, int blocks, cudaStream_t s);
cudaError_t launch_advance(const AdvanceArgs &a, cudaStream_t s);
cudaError_t launch_set_range_bits(uint32_t *vis, uint64_t v0, uint64_t v1, cudaStream_t s);
cudaError_t launch_fill_u32(uint32_t *p, uint32_t val, uint64_t n, cudaStream_t s);
int expand_occupancy(int mode);

}  // namespace efg
