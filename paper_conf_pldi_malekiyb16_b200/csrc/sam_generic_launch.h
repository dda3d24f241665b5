// sam_generic_launch.h -- host interface of the generic-operator / selectable-carry kernel
// (sam_generic.cu), used by the C ABI (sam_api.cu).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace sam {
namespace gen {

struct GenArgs {
    const void* in;
    void* out;
    uint64_t n;
    int s, k, inclusive, mode;  // mode: GEN_STATIC / GEN_LOOKBACK / GEN_CHAINED
    unsigned long long* words;  // workspace: tagged aggregate / inclusive words
    size_t words_bytes;
    unsigned long long* tile_ctr;
    unsigned int* done_ctr;
    unsigned int* epoch_ptr;
    int dev, num_sms;
    cudaStream_t stream;
    int* mode_used;  // out: the carry scheme that ran (the static one falls back to look-back)
};

// elem = sam_dtype (0 i32, 1 i64, 2 f32, 3 f64, 4 u32, 5 u64); op = sam_op
cudaError_t launch_generic(int elem, int op, const GenArgs& a);
// workspace bytes of tagged words for n elements
size_t generic_words_bytes(int elem, int k, int s, uint64_t n);

}  // namespace gen
}  // namespace sam
