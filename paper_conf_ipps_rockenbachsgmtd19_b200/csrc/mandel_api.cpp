// mandel_api.cpp -- C ABI of row NEXT-4 (include/mandel.h): launches of the
// batched Mandelbrot kernel (mandel.cu) and the streamed whole-image driver
// with round-robin memory spaces.
#include <cuda_runtime.h>

#include <chrono>
#include <vector>

#include "internal.h"
#include "mandel.h"

namespace {

bool valid_image(int32_t dim, int32_t niter) {
    return dim >= 1 && niter >= 1 && niter <= 8388607;  // k * 255 fits in int32
}

int device_sms(int dev) {
    int sms = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 0;
    return sms;
}

struct Space {
    int dev = 0;
    cudaStream_t s = nullptr;
    uint8_t* img = nullptr;
    uint32_t* counter = nullptr;
    uint64_t* iters = nullptr;
};

}  // namespace

extern "C" dedup_status mandel_rows_device(void* stream, int32_t dim, int32_t niter,
                                           double init_a, double init_b, double range,
                                           int32_t row0, int32_t nrows, uint8_t* d_img,
                                           uint32_t* d_counter, uint64_t* d_iters) {
    if (!valid_image(dim, niter) || row0 < 0 || nrows < 0 || row0 > dim || nrows > dim - row0)
        return DEDUP_EINVAL;
    if (nrows == 0) return DEDUP_OK;
    if (d_img == nullptr || d_counter == nullptr) return DEDUP_EINVAL;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return DEDUP_ECUDA;
    if (dd::mandel_unlaunchable()) return DEDUP_ECUDA;
    const double step = range / ((double)dim);  // Listing 1 line 3
    dd::launch_mandel(dim, niter, init_a, init_b, step, row0, nrows, d_img, d_counter, d_iters,
                      device_sms(dev), static_cast<cudaStream_t>(stream));
    return cudaGetLastError() == cudaSuccess ? DEDUP_OK : DEDUP_ECUDA;
}

extern "C" dedup_status mandel_image(const mandel_config* cfg, uint8_t* host_img,
                                     double* ms_out, uint64_t* iters_out) {
    if (cfg == nullptr || host_img == nullptr || !valid_image(cfg->dim, cfg->niter) ||
        cfg->batch_rows < 1 || cfg->spaces < 1 || cfg->spaces > 64 || cfg->num_devices < 1)
        return DEDUP_EINVAL;
    const int32_t dim = cfg->dim;
    const double step = cfg->range / ((double)dim);
    const uint32_t rows = cfg->batch_rows < (uint32_t)dim ? cfg->batch_rows : (uint32_t)dim;
    const size_t img_bytes = (size_t)dim * (size_t)dim;
    int prev = 0;
    cudaGetDevice(&prev);
    dedup_status st = DEDUP_OK;
    std::vector<Space> sp(cfg->spaces);
    bool registered = false;
    cudaError_t e = cudaHostRegister(host_img, img_bytes, cudaHostRegisterDefault);
    if (e == cudaSuccess) registered = true;
    else cudaGetLastError();  // already page-locked (or not registrable): plain copies
    for (uint32_t k = 0; k < cfg->spaces && st == DEDUP_OK; ++k) {
        const uint32_t d = k % cfg->num_devices;
        sp[k].dev = cfg->device_ids ? cfg->device_ids[d] : (int)d;
        if (cudaSetDevice(sp[k].dev) != cudaSuccess ||
            cudaStreamCreateWithFlags(&sp[k].s, cudaStreamNonBlocking) != cudaSuccess)
            st = DEDUP_ECUDA;
        else if (cudaMalloc(&sp[k].img, (size_t)rows * dim) != cudaSuccess ||
                 cudaMalloc(&sp[k].counter, sizeof(uint32_t)) != cudaSuccess ||
                 cudaMalloc(&sp[k].iters, sizeof(uint64_t)) != cudaSuccess ||
                 cudaMemset(sp[k].iters, 0, sizeof(uint64_t)) != cudaSuccess)
            st = DEDUP_ENOMEM;
        else if (dd::mandel_unlaunchable())
            st = DEDUP_ECUDA;
    }
    std::vector<int> sms(cfg->spaces);
    for (uint32_t k = 0; k < cfg->spaces && st == DEDUP_OK; ++k) sms[k] = device_sms(sp[k].dev);
    const auto t0 = std::chrono::steady_clock::now();
    for (int32_t row0 = 0, b = 0; row0 < dim && st == DEDUP_OK; row0 += (int32_t)rows, ++b) {
        Space& s = sp[(uint32_t)b % cfg->spaces];
        const int32_t n = dim - row0 < (int32_t)rows ? dim - row0 : (int32_t)rows;
        cudaSetDevice(s.dev);
        dd::launch_mandel(dim, cfg->niter, cfg->init_a, cfg->init_b, step, row0, n, s.img,
                          s.counter, iters_out ? s.iters : nullptr,
                          sms[(uint32_t)b % cfg->spaces], s.s);
        if (cudaMemcpyAsync(host_img + (size_t)row0 * dim, s.img, (size_t)n * dim,
                            cudaMemcpyDeviceToHost, s.s) != cudaSuccess)
            st = DEDUP_ECUDA;
    }
    for (auto& s : sp) {
        if (s.s == nullptr) continue;
        cudaSetDevice(s.dev);
        if (cudaStreamSynchronize(s.s) != cudaSuccess) st = DEDUP_ECUDA;
    }
    const auto t1 = std::chrono::steady_clock::now();
    if (ms_out) *ms_out = std::chrono::duration<double, std::milli>(t1 - t0).count();
    if (iters_out) {
        *iters_out = 0;
        for (auto& s : sp) {
            uint64_t v = 0;
            cudaSetDevice(s.dev);
            if (s.iters && st == DEDUP_OK &&
                cudaMemcpy(&v, s.iters, sizeof(v), cudaMemcpyDeviceToHost) == cudaSuccess)
                *iters_out += v;
        }
    }
    for (auto& s : sp) {
        cudaSetDevice(s.dev);
        if (s.img) cudaFree(s.img);
        if (s.counter) cudaFree(s.counter);
        if (s.iters) cudaFree(s.iters);
        if (s.s) cudaStreamDestroy(s.s);
    }
    if (registered) cudaHostUnregister(host_img);
    cudaSetDevice(prev);
    if (st == DEDUP_OK && cudaGetLastError() != cudaSuccess) st = DEDUP_ECUDA;
    return st;
}
