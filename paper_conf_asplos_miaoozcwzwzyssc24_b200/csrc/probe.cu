// probe.cu — measurement kernel: the practical HBM read ceiling of the same bytes
// the attention kernel streams, read the way it reads them (bulk async copies into a shared-memory
// ring, one issuing thread per CTA, persistent grid of one CTA per SM) with no compute at all.
// bench.py reports the attention kernel's bandwidth against this ceiling next to the copy peak.
#include "common.cuh"

namespace specinfer {

constexpr int kProbeChunk = 32768;   // bytes per bulk copy (one K or V tile of the attention kernel)
constexpr int kProbeSlots = 6;       // copies in flight per CTA (the attention kernel's 3 K + 3 V)

__global__ void __launch_bounds__(32, 1) hbm_read_probe_kernel(const uint8_t *__restrict__ src, size_t bytes) {
    extern __shared__ __align__(128) uint8_t ring[];
    __shared__ uint64_t full[kProbeSlots];
    if (threadIdx.x != 0) return;
    // this CTA's contiguous share, in whole chunks (the last CTA takes the remainder)
    const size_t chunks = (bytes + kProbeChunk - 1) / kProbeChunk;
    const size_t c0 = chunks * blockIdx.x / gridDim.x, c1 = chunks * (blockIdx.x + 1) / gridDim.x;
    for (int i = 0; i < kProbeSlots; ++i) mbar_init(&full[i], 1);
    fence_barrier_init();
    size_t issued = c0;
    auto issue = [&](int slot) {
        const size_t off = issued * kProbeChunk;
        const uint32_t n = (uint32_t)min((size_t)kProbeChunk, bytes - off);
        mbar_arrive_expect_tx(&full[slot], n);
        bulk_load_g2s(ring + (size_t)slot * kProbeChunk, src + off, n, &full[slot]);
        ++issued;
    };
    for (int i = 0; i < kProbeSlots && issued < c1; ++i) issue(i);
    for (size_t c = c0; c < c1; ++c) {
        const int slot = (int)((c - c0) % kProbeSlots);
        mbar_wait(&full[slot], (uint32_t)(((c - c0) / kProbeSlots) & 1));
        if (issued < c1) issue(slot);
    }
}

cudaError_t launch_hbm_read_probe(const void *src, size_t bytes, int num_sms, cudaStream_t stream) {
    if (bytes == 0) return cudaSuccess;
    const size_t smem = (size_t)kProbeSlots * kProbeChunk;
    cudaError_t e = cudaFuncSetAttribute(hbm_read_probe_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    hbm_read_probe_kernel<<<num_sms, 32, smem, stream>>>(reinterpret_cast<const uint8_t *>(src), bytes);
    return cudaGetLastError();
}

}  // namespace specinfer
