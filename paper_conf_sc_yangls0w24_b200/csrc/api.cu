// api.cu — error model and small entry points of the C ABI (include/xbfs.h).
#include <stdarg.h>
#include <stdio.h>
#include <string.h>

#include "common.cuh"

namespace xbfs {

static thread_local char g_err[512] = "";

xbfs_status set_error(xbfs_status s, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return s;
}

xbfs_status cuda_fail(xbfs_graph* g, cudaError_t e, const char* what) {
    if (g) g->poisoned = true;
    if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();
        return set_error(XBFS_ERR_OUT_OF_MEMORY, "out of device memory in %s", what);
    }
    return set_error(XBFS_ERR_CUDA, "CUDA error %d (%s) in %s", (int)e, cudaGetErrorString(e), what);
}

}  // namespace xbfs

xbfs::KArgs xbfs_graph::kargs() const {
    xbfs::KArgs a;
    long long words = (n + 31) / 32;
    a.row_ptr = row_ptr;
    a.col = col;
    a.level = nullptr;
    a.parent = nullptr;
    a.head = head;
    a.head32 = head32;
    a.idbits = idbits;
    a.visited = visited;
    const long long stride = (words + 31) / 32 * 32;  // 128-byte aligned bitmaps (uint4 access)
    for (int i = 0; i < 3; ++i) a.fb[i] = fb + i * stride;
    a.la = fb + 3 * stride;
    for (int i = 0; i < 3; ++i) {
        a.qv[i] = qv + i * n;
        a.qoff[i] = qoff + i * n;
        a.qdelta[i] = qdelta + i * n;
        a.tile_first[i] = tile_first + i * tiles_cap;
    }
    a.st = st;
    a.hctl = hctl_dev;
    a.log = log;
    a.n = n;
    a.words = words;
    a.arcs = arcs;
    a.dbits = dbits;
    a.track_max = 1;
    a.directed = directed;
    a.bu_row_ptr = directed ? in_row_ptr : row_ptr;
    a.bu_col = directed ? in_col : col;
    a.bu_head32 = directed ? in_head32 : head32;
    return a;
}

extern "C" {

const char* xbfs_last_error(void) { return xbfs::g_err; }

int32_t xbfs_compiled_arch(void) {
#ifdef XBFS_ARCH
    return XBFS_ARCH;
#else
    return 0;
#endif
}

void xbfs_run_opts_default(xbfs_run_opts* o) {
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->alpha = 0.04;      // P:L347 gives 0.1 (MI250X); re-tuned on B200 (reading C-13,
                          // tools/sweep_selector.py, profiles/r01_selector_sweep.md)
    o->grow = 2.0;        // reading C-10
    o->ratio_min = 1e-3;  // reading C-10
    o->bu_stay = 1.0;     // reading C-11, tuned on B200 (tools/sweep_selector.py); 0 = paper rule
    o->force_strategy = -1;
    o->small_edges = 65536;  // small-frontier cluster mode threshold (tuned on the grid config)
    o->driver = 0;
}

xbfs_status xbfs_graph_info(const xbfs_graph* g, int64_t* n, int64_t* arcs, int64_t* input_edges,
                            int32_t* max_degree) {
    if (!g) return xbfs::set_error(XBFS_ERR_INVALID_ARG, "xbfs_graph_info: NULL handle");
    if (n) *n = g->n;
    if (arcs) *arcs = g->arcs;
    if (input_edges) *input_edges = g->m_input;
    if (max_degree) *max_degree = g->max_deg;
    return XBFS_OK;
}

xbfs_status xbfs_copy_csr(const xbfs_graph* gc, int64_t* row_ptr_host, int32_t* col_host) {
    xbfs_graph* g = const_cast<xbfs_graph*>(gc);
    if (!g || !row_ptr_host || (!col_host && g->arcs > 0))
        return xbfs::set_error(XBFS_ERR_INVALID_ARG, "xbfs_copy_csr: NULL argument");
    if (g->poisoned) return xbfs::set_error(XBFS_ERR_STATE, "handle poisoned by an earlier failure");
    if (g->dist) return xbfs::set_error(XBFS_ERR_STATE, "xbfs_copy_csr: distributed handle");
    XBFS_CUDA(g, cudaSetDevice(g->device));
    XBFS_CUDA(g, cudaMemcpyAsync(row_ptr_host, g->row_ptr, (g->n + 1) * sizeof(long long),
                                 cudaMemcpyDeviceToHost, g->stream));
    if (g->arcs > 0)
        XBFS_CUDA(g, cudaMemcpyAsync(col_host, g->col, g->arcs * sizeof(int), cudaMemcpyDeviceToHost,
                                     g->stream));
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    return XBFS_OK;
}

void xbfs_destroy(xbfs_graph* g) {
    if (!g) return;
    cudaSetDevice(g->device);
    if (g->stream) cudaStreamSynchronize(g->stream);
    if (g->copy_stream) cudaStreamSynchronize(g->copy_stream);
    if (g->dist) xbfs::dist_destroy(g->dist);
    if (g->loop_exec) cudaGraphExecDestroy(g->loop_exec);
    void* dev[] = {g->row_ptr, g->col, g->tcount, g->nonisolated, g->visited, g->fb, g->qv,
                   g->qoff, g->qdelta, g->tile_first, g->st, g->log, g->red_scratch,
                   g->scratch_level, g->scratch_parent, g->head, g->head32,
                   g->in_row_ptr, g->in_col, g->in_head32};
    for (void* p : dev)
        if (p) cudaFree(p);
    if (g->hctl) cudaFreeHost(g->hctl);
    if (g->hstage) cudaFreeHost(g->hstage);
    for (cudaEvent_t e : g->ev_stage)
        if (e) cudaEventDestroy(e);
    if (g->ev0) cudaEventDestroy(g->ev0);
    if (g->ev1) cudaEventDestroy(g->ev1);
    for (cudaEvent_t e : g->prof_events) cudaEventDestroy(e);
    for (int s = 0; s < 2; ++s) {
        if (g->ev_done[s]) cudaEventDestroy(g->ev_done[s]);
        if (g->ev_copied[s]) cudaEventDestroy(g->ev_copied[s]);
    }
    if (g->copy_stream) cudaStreamDestroy(g->copy_stream);
    cudaGetLastError();
    delete g;
}

}  // extern "C"
