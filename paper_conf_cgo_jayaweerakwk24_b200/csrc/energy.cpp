// energy.cpp -- NVML energy harness and the tile-space sweep.
//
// The paper samples nvidia-smi power every 10 ms, runs each variant 100 times
// and estimates energy = P_avg * t_exec; PPW = FLOP/s / W.
// On B200 we read NVML's total-energy counter (mJ since driver load) around a
// window of back-to-back runs -- the integral the paper approximates -- and keep
// a 10 ms sampler of power and SM clock alongside (the paper's cadence).
// NVML is loaded with dlopen so the library has no link-time NVML dependency;
// when it is missing the energy calls return EATSS_E_NVML and the sweep still
// reports times.  Clocks are never locked (the effect relies on DVFS).
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstring>
#include <mutex>
#include <thread>
#include <vector>

#include "desc.hpp"

namespace eatss {

namespace {
typedef int nvmlReturn_t;
typedef void *nvmlDevice_t;
struct Nvml {
    void *h = nullptr;
    bool ok = false;
    nvmlReturn_t (*init)(void) = nullptr;
    nvmlReturn_t (*by_pci)(const char *, nvmlDevice_t *) = nullptr;
    nvmlReturn_t (*by_index)(unsigned, nvmlDevice_t *) = nullptr;
    nvmlReturn_t (*energy)(nvmlDevice_t, unsigned long long *) = nullptr;
    nvmlReturn_t (*power)(nvmlDevice_t, unsigned *) = nullptr;
    nvmlReturn_t (*clock)(nvmlDevice_t, int, unsigned *) = nullptr;
};

Nvml &nvml() {
    static Nvml n;
    static std::once_flag once;
    std::call_once(once, [] {
        const char *names[] = {"libnvidia-ml.so.1", "libnvidia-ml.so"};
        for (const char *nm : names)
            if ((n.h = dlopen(nm, RTLD_NOW | RTLD_LOCAL))) break;
        if (!n.h) return;
        n.init = (nvmlReturn_t(*)(void))dlsym(n.h, "nvmlInit_v2");
        n.by_pci = (nvmlReturn_t(*)(const char *, nvmlDevice_t *))dlsym(n.h, "nvmlDeviceGetHandleByPciBusId_v2");
        n.by_index = (nvmlReturn_t(*)(unsigned, nvmlDevice_t *))dlsym(n.h, "nvmlDeviceGetHandleByIndex_v2");
        n.energy = (nvmlReturn_t(*)(nvmlDevice_t, unsigned long long *))dlsym(n.h, "nvmlDeviceGetTotalEnergyConsumption");
        n.power = (nvmlReturn_t(*)(nvmlDevice_t, unsigned *))dlsym(n.h, "nvmlDeviceGetPowerUsage");
        n.clock = (nvmlReturn_t(*)(nvmlDevice_t, int, unsigned *))dlsym(n.h, "nvmlDeviceGetClockInfo");
        n.ok = n.init && n.energy && n.power && n.clock && (n.by_pci || n.by_index) && n.init() == 0;
    });
    return n;
}

// NVML handle of a CUDA device ordinal (matched by PCI bus id: CUDA_VISIBLE_DEVICES safe)
bool handle(int device, nvmlDevice_t *out) {
    Nvml &n = nvml();
    if (!n.ok) return false;
    char bus[64] = {0};
    if (n.by_pci && cudaDeviceGetPCIBusId(bus, sizeof(bus), device) == cudaSuccess &&
        n.by_pci(bus, out) == 0)
        return true;
    return n.by_index && n.by_index((unsigned)device, out) == 0;
}

struct Sampler {
    std::atomic<bool> stop{false};
    std::vector<unsigned> mw, mhz;
    std::thread th;
    void start(nvmlDevice_t h) {
        th = std::thread([this, h] {
            Nvml &n = nvml();
            while (!stop.load()) {
                unsigned p = 0, c = 0;
                if (n.power(h, &p) == 0) mw.push_back(p);
                if (n.clock(h, 1 /*NVML_CLOCK_SM*/, &c) == 0) mhz.push_back(c);
                std::this_thread::sleep_for(std::chrono::milliseconds(10));
            }
        });
    }
    void finish() {
        stop = true;
        if (th.joinable()) th.join();
    }
};

double median(std::vector<unsigned> v) {
    if (v.empty()) return 0;
    std::sort(v.begin(), v.end());
    return v[v.size() / 2];
}
}  // namespace

}  // namespace eatss

using namespace eatss;

extern "C" eatss_status eatss_energy_mj(int device, uint64_t *mj) {
    if (!mj) return fail(EATSS_E_INVALID, "eatss_energy_mj: null");
    nvmlDevice_t h;
    if (!handle(device, &h)) return fail(EATSS_E_NVML, "NVML unavailable");
    unsigned long long v = 0;
    if (nvml().energy(h, &v) != 0) return fail(EATSS_E_NVML, "nvmlDeviceGetTotalEnergyConsumption failed");
    *mj = v;
    return EATSS_OK;
}

extern "C" eatss_status eatss_power_sample(int device, uint32_t *mw, uint32_t *sm_mhz) {
    nvmlDevice_t h;
    if (!handle(device, &h)) return fail(EATSS_E_NVML, "NVML unavailable");
    unsigned p = 0, c = 0;
    if (mw && nvml().power(h, &p) != 0) return fail(EATSS_E_NVML, "nvmlDeviceGetPowerUsage failed");
    if (sm_mhz && nvml().clock(h, 1 /*NVML_CLOCK_SM*/, &c) != 0) return fail(EATSS_E_NVML, "nvmlDeviceGetClockInfo failed");
    if (mw) *mw = p;
    if (sm_mhz) *sm_mhz = c;
    return EATSS_OK;
}

extern "C" eatss_status eatss_sweep(const eatss_kernel_desc *d, const int64_t *variants, int n,
                                    void *const *buffers, int device, int warmup, double min_window_s,
                                    eatss_measurement *results) {
    if (!d || !variants || !buffers || !results || n < 0)
        return fail(EATSS_E_INVALID, "eatss_sweep: null argument");
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return fail(EATSS_E_CUDA, std::string("cudaSetDevice: ") + cudaGetErrorString(e));
    const int L = eatss_desc_num_loops(d);
    const double flops = eatss_desc_flops(d);
    cudaStream_t s;
    if ((e = cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking)) != cudaSuccess)
        return fail(EATSS_E_CUDA, "cudaStreamCreate failed");
    cudaEvent_t ev0, ev1;
    cudaEventCreate(&ev0);
    cudaEventCreate(&ev1);
    nvmlDevice_t h = nullptr;
    const bool have_nvml = handle(device, &h);
    for (int v = 0; v < n; v++) {
        eatss_measurement &r = results[v];
        std::memset(&r, 0, sizeof(r));
        const int64_t *t = variants + (int64_t)v * L;
        eatss_status st = EATSS_OK;
        for (int w = 0; w < std::max(1, warmup) && st == EATSS_OK; w++) st = eatss_run(d, t, buffers, s);
        if (st != EATSS_OK || cudaStreamSynchronize(s) != cudaSuccess) {
            r.status = st != EATSS_OK ? st : EATSS_E_CUDA;
            cudaGetLastError();
            continue;
        }
        // one timed run sizes the window
        cudaEventRecord(ev0, s);
        eatss_run(d, t, buffers, s);
        cudaEventRecord(ev1, s);
        cudaEventSynchronize(ev1);
        float ms1 = 0;
        cudaEventElapsedTime(&ms1, ev0, ev1);
        // The NVML energy counter updates in steps (~100 ms on B200, calibrated by the
        // harness), so the window is ALIGNED to counter updates: the device is kept busy
        // with chunks of runs; the window opens at one update and closes at the first
        // update after min_window_s.  P_avg = dE / dt over that window, and the
        // energy per run = P_avg * t_run with t_run from CUDA events inside the window.
        const int64_t chunk = std::max<int64_t>(1, (int64_t)std::ceil(10.0 / std::max(ms1, 1e-3f)));
        constexpr int Q = 4;  // chunk events in flight (3 queued ahead)
        cudaEvent_t cev[Q];
        for (int i = 0; i < Q; i++) cudaEventCreateWithFlags(&cev[i], cudaEventDisableTiming);
        int64_t launched = 0, inflight = 0, head = 0;
        auto launch_chunk = [&]() {
            for (int64_t k = 0; k < chunk && st == EATSS_OK; k++) st = eatss_run(d, t, buffers, s);
            cudaEventRecord(cev[head % Q], s);
            head++;
            inflight++;
            launched += chunk;
        };
        auto pump = [&]() {
            while (inflight > 0 && cudaEventQuery(cev[(head - inflight) % Q]) == cudaSuccess) inflight--;
            while (inflight < Q - 1 && st == EATSS_OK) launch_chunk();
        };
        using clk = std::chrono::steady_clock;
        Sampler smp;
        unsigned long long ea = 0, eb = 0, cur = 0;
        clk::time_point ta, tb;
        int64_t runs_a = 0, runs_b = 0;
        pump();
        if (have_nvml) {
            smp.start(h);
            nvml().energy(h, &cur);
            const unsigned long long start = cur;
            const auto t_guard = clk::now();
            while (cur == start && st == EATSS_OK &&
                   std::chrono::duration<double>(clk::now() - t_guard).count() < 2.0) {
                pump();
                std::this_thread::sleep_for(std::chrono::microseconds(200));
                nvml().energy(h, &cur);
            }
            ea = cur;
        }
        ta = clk::now();
        cudaEventRecord(ev0, s);  // start of the timed runs (launched from here on)
        runs_a = launched;
        while (st == EATSS_OK) {
            pump();
            const double el = std::chrono::duration<double>(clk::now() - ta).count();
            // the window must contain at least one run launched after ta (a variant slower than the window
            // would otherwise close it with only the runs queued before ta in flight: zero timed runs)
            if (el >= min_window_s && launched > runs_a) {
                if (!have_nvml) break;
                nvml().energy(h, &cur);
                if (cur != ea && cur != eb) {
                    if (eb == 0) eb = cur;  // first update after the minimum window closes it
                }
                if (eb != 0) break;
                if (el > min_window_s + 2.0 + 4.0 * ms1 * 1e-3) break;  // counter stalled: give up on energy
            }
            std::this_thread::sleep_for(std::chrono::microseconds(200));
        }
        tb = clk::now();
        runs_b = launched;
        cudaEventRecord(ev1, s);
        cudaError_t se = cudaEventSynchronize(ev1);
        if (have_nvml) smp.finish();
        for (int i = 0; i < Q; i++) cudaEventDestroy(cev[i]);
        if (st != EATSS_OK || se != cudaSuccess) {
            r.status = st != EATSS_OK ? st : EATSS_E_CUDA;
            cudaGetLastError();
            continue;
        }
        float ms = 0;
        cudaEventElapsedTime(&ms, ev0, ev1);
        const int64_t runs = std::max<int64_t>(1, runs_b - runs_a);
        r.runs = runs;
        r.ms_per_run = ms / runs;
        r.tflops = flops / (r.ms_per_run * 1e-3) / 1e12;
        const double win_s = std::chrono::duration<double>(tb - ta).count();
        if (have_nvml && eb > ea && win_s > 0) {
            r.avg_watts = (double)(eb - ea) * 1e-3 / win_s;
            r.joules_per_run = r.avg_watts * r.ms_per_run * 1e-3;
            r.gflops_per_watt = flops / r.joules_per_run / 1e9;  // FLOP/J == (FLOP/s)/W
        }
        r.sm_mhz_median = median(smp.mhz);
        r.status = (have_nvml && eb > ea) ? EATSS_OK : EATSS_E_NVML;
    }
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
    cudaStreamDestroy(s);
    return EATSS_OK;
}
