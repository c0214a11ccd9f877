// simd_group.cuh -- a2: the SIMD-group partition of a team and its queries.
//
// "the team of threads is evenly divided into SIMD groups,
// where all threads within a group occupy the same warp ... One thread in each
// group is designated as the SIMD main thread".  PAPER.md:255-258: a simd
// loop runs on "a set of adjacent threads".  The runtime queries of
// PAPER.md:507-529 map one-to-one onto a statically sized cooperative-groups
// tile of `S` adjacent lanes (a warp is never split across groups because
// S divides 32):
//   getSimdGroup      -> tile.meta_group_rank()      (= threadIdx.x / S)
//   getSimdGroupId    -> tile.thread_rank()          (= threadIdx.x % S; main = 0)
//   getSimdGroupSize  -> S                           (compile-time, per launch)
//   isSimdGroupLeader -> thread_rank() == 0
//   simdmask          -> lanes of this warp in the group: ((1<<S)-1) << (lane & ~(S-1))
//   synchronizeWarp   -> tile.sync() == __syncwarp(simdmask())
#pragma once

#include <cooperative_groups.h>
#include <cstdint>

namespace nest {
namespace cg = cooperative_groups;

// WU ("warp-uniform"): the caller guarantees that every lane of the warp
// reaches each collective of the group together (all groups of the warp run
// the same number of batches), so the data exchanges use the full-warp mask
// -- xor offsets < S never leave the group, results are identical -- and skip
// the sub-warp convergence checks, and synchronizeWarp(simdmask()) becomes a
// full-warp __syncwarp(): with every lane of the warp at the same barrier it
// orders exactly what the group barrier would (a superset of the group).
template <int S, bool WU = false>
struct SimdGroup {
    static_assert(S == 1 || S == 2 || S == 4 || S == 8 || S == 16 || S == 32,
                  "simdlen must divide the warp (PAPER.md:484-491)");
    cg::thread_block_tile<S, cg::thread_block> tile;

    __device__ __forceinline__ SimdGroup() : tile(cg::tiled_partition<S>(cg::this_thread_block())) {}

    __device__ __forceinline__ int group() const { return (int)tile.meta_group_rank(); }   // getSimdGroup
    __device__ __forceinline__ int id() const { return (int)tile.thread_rank(); }          // getSimdGroupId
    static constexpr int size() { return S; }                                              // getSimdGroupSize
    __device__ __forceinline__ bool leader() const { return tile.thread_rank() == 0; }     // isSimdGroupLeader
    __device__ __forceinline__ unsigned mask() const {                                     // simdmask
        if constexpr (S == 32) {
            return 0xffffffffu;
        } else {
            const unsigned lane = threadIdx.x & 31u;
            return ((1u << S) - 1u) << (lane & ~unsigned(S - 1));
        }
    }
    __device__ __forceinline__ void sync() const {                                         // synchronizeWarp
        if constexpr (S == 1) {
            return;
        } else if constexpr (WU) {
            __syncwarp();   // every lane of the warp is here: the group barrier is implied
        } else {
            tile.sync();
        }
    }
    template <class T>
    __device__ __forceinline__ T bcast(T v) const {                                       // lane 0 -> group
        if constexpr (S == 1) {
            return v;
        } else if constexpr (WU) {
            return __shfl_sync(0xffffffffu, v, 0, S);
        } else {
            return tile.shfl(v, 0);
        }
    }
    template <class T>
    __device__ __forceinline__ T shfl_xor(T v, unsigned m) const {
        if constexpr (S == 1) {
            return v;
        } else if constexpr (WU) {
            return __shfl_xor_sync(0xffffffffu, v, m);
        } else {
            return tile.shfl_xor(v, m);
        }
    }
};

}  // namespace nest
