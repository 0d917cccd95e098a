// desc.hpp -- internal kernel descriptor of libeatss (not part of the ABI).
//
// A descriptor holds (a) the affine program as the model sees it -- nests of
// loops and array references ("reference f^A", P:133 subscripts,
// P:177 parallel/serial loops) -- and (b) what the executor needs: the builtin
// kind, extents, dtype, scalars, execution options and cached CUDA graphs.
#pragma once

#include <cstdint>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/eatss.h"

namespace eatss {

// One array subscript: the set of loop positions (bitmask over the nest's
// depth positions) that appear in it, plus a constant offset (halo).
struct Sub {
    uint32_t iters = 0;
    int32_t off = 0;
};

struct Ref {
    int array = 0;  // array id within the program
    std::vector<Sub> subs;
    bool write = false;
};

struct Loop {
    int64_t extent = 0;
    bool parallel = true;
};

struct Nest {
    std::vector<Loop> loops;  // outermost first; position p <-> tile entry p
    std::vector<Ref> refs;
};

struct GraphKey {
    std::vector<int64_t> tiles;
    std::vector<uintptr_t> bufs;
    uintptr_t stream;
    bool operator<(const GraphKey &o) const {
        if (tiles != o.tiles) return tiles < o.tiles;
        if (bufs != o.bufs) return bufs < o.bufs;
        return stream < o.stream;
    }
};

}  // namespace eatss

struct eatss_kernel_desc {
    eatss_builtin kind;
    eatss_dtype dtype;
    std::vector<int64_t> dims;
    int64_t tsteps = 0;
    double alpha = 1.5, beta = 1.2;
    eatss_exec_opts exec{50, EATSS_ENGINE_AUTO, 1, 0, 0, 0};
    std::vector<eatss::Nest> nests;
    int num_buffers = 0;
    std::vector<int64_t> buffer_elems;
    // cached stencil time-loop graphs (cudaGraphExec_t as void*)
    std::mutex graph_mu;
    std::map<eatss::GraphKey, void *> graphs;
    std::map<eatss::GraphKey, int> graph_cvs;  // carve-out each graph's launches were captured with
    int graph_cv = -1;                         // carve-out of the last stencil issue / replay
    // exec.time_kernels: start/stop events per nest of the last timed run (cudaEvent_t as void*)
    std::vector<void *> kev;
    int kev_dev = -1, kev_valid = 0;
    // carve-out (percent) requested by each nest's main kernel in the last run (-1: none)
    std::vector<int> last_cv;
    // eatss_run_host: library-owned device copies of the buffers, copy streams and events
    std::vector<void *> hbuf;
    std::vector<size_t> hbuf_bytes;
    int hdev = -1;
    void *hstream[2] = {nullptr, nullptr};  // host->device, device->host
    std::vector<void *> hev;                // pipeline events
    // library-owned scratch (mttkrp split-k partials), grown on demand, freed with the descriptor
    void *ws = nullptr;
    size_t ws_bytes = 0;
    int ws_dev = -1;
    ~eatss_kernel_desc();
};

namespace eatss {

// thread-local error message
void set_error(const std::string &msg);
eatss_status fail(eatss_status s, const std::string &msg);

// model (model.cpp)
struct NestModel {
    int nrefs = 0;
    int ls1 = 0;                      // position of l_s1
    std::vector<int> cnt;             // per position
    std::vector<uint32_t> l1_fp;      // footprints (iterator bitmasks) in L1_set
    std::vector<uint32_t> sh_fp;      // footprints in SH_set (L1 duplicates dropped)
    uint32_t bset = 0;                // bitmask of B-set positions
    std::vector<int64_t> H;           // per position
};
NestModel derive_nest(const Nest &n, int waf);
std::vector<int64_t> program_extents(const eatss_kernel_desc &d);

inline int dtype_bytes(eatss_dtype t) { return t == EATSS_F64 ? 8 : 4; }

}  // namespace eatss
