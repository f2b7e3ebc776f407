// faults.cu -- seeded fault sites and bit-flip injection for FT2's fault
// models (1-bit, 2-bit, EXP; L88: one fault per inference; L90:
// site = layer ID, neuron ID, bit location; L95: uniform over the linear
// layers of the decoder blocks).  Site generation follows reading R6 exactly
// (Philox4x32-10 keyed by the seed, counter = trial id), so any trial range
// can be generated on any GPU and agrees bit for bit with the CPU oracle.
#include <cuda_runtime.h>

#include "ft2_device.cuh"
#include "ft2_internal.h"

namespace ft2impl {
using namespace ft2dev;

struct SitesK {
    uint64_t seed, trial0;
    int32_t n, model, dtype;
    int32_t n_steps, prompt_len, n_layers, layer_uniform, step_policy;
    uint64_t total_neurons;
    int32_t width[FT2_MAX_SITE_LAYERS];
};

__global__ void make_sites_kernel(const __grid_constant__ SitesK p, ft2_fault_site* out) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= p.n) return;
    uint64_t t = p.trial0 + (uint64_t)i;
    uint32_t k0 = (uint32_t)p.seed, k1 = (uint32_t)(p.seed >> 32);
    u32x4 u = philox4x32_10(u32x4{(uint32_t)t, (uint32_t)(t >> 32), 0u, 0x46543200u}, k0, k1);
    u32x4 v = philox4x32_10(u32x4{(uint32_t)t, (uint32_t)(t >> 32), 1u, 0x46543200u}, k0, k1);
    const uint32_t width_bits = p.dtype == FT2_FP32 ? 32u : 16u;
    const uint32_t exp_lo = p.dtype == FT2_BF16 ? 7u : (p.dtype == FT2_FP16 ? 10u : 23u);
    const uint32_t exp_n = p.dtype == FT2_FP16 ? 5u : 8u;
    ft2_fault_site s;
    s.trial = (uint32_t)t;
    uint32_t step = p.step_policy == 1 ? 1u + (uint32_t)(t % (uint64_t)p.n_steps)
                                       : draw_below(u.x, (uint32_t)p.n_steps + 1u);
    s.step = (uint16_t)step;
    uint32_t layer, col;
    if (p.layer_uniform) {
        layer = draw_below(u.y, (uint32_t)p.n_layers);
        col = draw_below(u.z, (uint32_t)p.width[layer]);
    } else {
        uint64_t g = ((uint64_t)u.y * p.total_neurons) >> 32;
        layer = 0;
        while (g >= (uint64_t)p.width[layer]) { g -= (uint64_t)p.width[layer]; ++layer; }
        col = (uint32_t)g;
    }
    s.layer = (uint16_t)layer;
    s.col = col;
    s.token = step == 0 ? draw_below(v.x, (uint32_t)p.prompt_len) : 0u;
    uint32_t mask;
    if (p.model == FT2_FAULT_1BIT) {
        mask = 1u << draw_below(u.w, width_bits);
        s.nbits = 1;
    } else if (p.model == FT2_FAULT_2BIT) {
        uint32_t b1 = draw_below(u.w, width_bits);
        uint32_t b2p = draw_below(v.y, width_bits - 1u);
        uint32_t b2 = b2p + (b2p >= b1 ? 1u : 0u);
        mask = (1u << b1) | (1u << b2);
        s.nbits = 2;
    } else {
        mask = 1u << (exp_lo + draw_below(u.w, exp_n));
        s.nbits = 1;
    }
    s.xor_mask = mask;
    s.model = (uint8_t)p.model;
    s.pad[0] = s.pad[1] = 0;
    out[i] = s;
}

__global__ void inject_kernel(uint16_t* y, int64_t rows, int64_t n, int64_t ld, const ft2_fault_site* sites,
                              int32_t n_sites, int32_t layer, int32_t step, const int32_t* base_row) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_sites) return;
    ft2_fault_site s = sites[i];
    if ((int32_t)s.step != step || (int32_t)s.layer != layer) return;
    int64_t row = (base_row ? (int64_t)base_row[i] : (int64_t)i) + (step == 0 ? (int64_t)s.token : 0);
    if (row < 0 || row >= rows || (int64_t)s.col >= n) return;
    y[row * ld + s.col] ^= (uint16_t)s.xor_mask;
}

cudaError_t launch_make_sites(uint64_t seed, uint64_t trial0, int32_t n, int32_t model, int32_t dtype,
                              const ft2_site_geometry& g, ft2_fault_site* out, cudaStream_t st, int* n_launch) {
    SitesK p;  // ~4 KB parameter block, built on the host per call
    p.seed = seed;
    p.trial0 = trial0;
    p.n = n;
    p.model = model;
    p.dtype = dtype;
    p.n_steps = g.n_steps;
    p.prompt_len = g.prompt_len;
    p.n_layers = g.n_layers;
    p.layer_uniform = g.layer_uniform;
    p.step_policy = g.step_policy;
    p.total_neurons = 0;
    for (int l = 0; l < g.n_layers; ++l) {
        p.width[l] = g.layer_width[l];
        p.total_neurons += (uint64_t)g.layer_width[l];
    }
    make_sites_kernel<<<(n + 127) / 128, 128, 0, st>>>(p, out);
    ++*n_launch;
    return cudaGetLastError();
}

cudaError_t launch_inject(uint16_t* y, int64_t rows, int64_t n, int64_t ld, const ft2_fault_site* sites,
                          int32_t n_sites, int32_t layer, int32_t step, const int32_t* base_row, cudaStream_t st,
                          int* n_launch) {
    inject_kernel<<<(n_sites + 127) / 128, 128, 0, st>>>(y, rows, n, ld, sites, n_sites, layer, step, base_row);
    ++*n_launch;
    return cudaGetLastError();
}

}  // namespace ft2impl
