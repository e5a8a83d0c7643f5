// C-ABI glue of libtdfs.so: status strings, thread-local error detail, option
// defaults, workspace sizing and the count / enumerate entry points (tdfs.h).
#include <cuda_runtime.h>

#include <cstdio>
#include <cstring>
#include <string>

#include "internal.h"

namespace tdfs {
namespace {
thread_local std::string g_last_error;
}
void set_error(const std::string& msg) { g_last_error = msg; }
int fail(int status, const std::string& msg) {
  g_last_error = msg;
  return status;
}
const char* last_error_cstr() { return g_last_error.c_str(); }
}  // namespace tdfs

using namespace tdfs;

extern "C" const char* tdfs_status_string(int s) {
  switch (s) {
    case TDFS_OK: return "TDFS_OK";
    case TDFS_E_INVALID_ARG: return "TDFS_E_INVALID_ARG";
    case TDFS_E_GRAPH_FORMAT: return "TDFS_E_GRAPH_FORMAT";
    case TDFS_E_ID_RANGE: return "TDFS_E_ID_RANGE";
    case TDFS_E_QUERY_DISCONNECTED: return "TDFS_E_QUERY_DISCONNECTED";
    case TDFS_E_QUERY_TOO_LARGE: return "TDFS_E_QUERY_TOO_LARGE";
    case TDFS_E_LABEL_RANGE: return "TDFS_E_LABEL_RANGE";
    case TDFS_E_OOM: return "TDFS_E_OOM";
    case TDFS_E_STACK_EXHAUSTED: return "TDFS_E_STACK_EXHAUSTED";
    case TDFS_E_OUTPUT_OVERFLOW: return "TDFS_E_OUTPUT_OVERFLOW";
    case TDFS_E_CUDA: return "TDFS_E_CUDA";
    case TDFS_E_WORKSPACE: return "TDFS_E_WORKSPACE";
    default: return "TDFS_E_UNKNOWN";
  }
}

extern "C" const char* tdfs_last_error(void) { return last_error_cstr(); }

extern "C" int tdfs_abi_version(void) { return TDFS_ABI_VERSION; }

extern "C" void tdfs_run_opts_default(tdfs_run_opts* o) {
  if (!o) return;
  std::memset(o, 0, sizeof(*o));
  o->tau_ns = 10 * 1000 * 1000;   // tau = 10 ms
  o->chunk = 8;
  o->queue_ints = 3000000;        // N = 3 M ints
  o->page_bytes = 8192;           // 8 KB pages
  o->page_table_entries = 0;      // auto from d_max (R15)
  o->pool_bytes = 0;              // auto
  o->blocks = 0;
  o->warps_per_block = 0;
  o->shard_rank = 0;
  o->shard_world = 1;
  o->flags = 0;
}

extern "C" size_t tdfs_workspace_bytes(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o) {
  tdfs_run_opts d;
  if (!o) {
    tdfs_run_opts_default(&d);
    o = &d;
  }
  WsLayout L;
  if (resolve_layout(graph_of(g), plan_of(p), o, &L) != TDFS_OK) return 0;
  return L.total;
}

extern "C" int tdfs_count(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                          size_t ws_bytes, void* stream, uint64_t* d_count, uint64_t* h_count, tdfs_stats* stats) {
  if (!g || !p) return fail(TDFS_E_INVALID_ARG, "count: NULL graph or plan");
  tdfs_run_opts d;
  if (!o) {
    tdfs_run_opts_default(&d);
    o = &d;
  }
  return launch_job(graph_of(g), plan_of(p), o, workspace, ws_bytes, stream, 0, nullptr, 0, d_count,
                    h_count != nullptr, h_count, stats, nullptr, 0, nullptr);
}

extern "C" int tdfs_enumerate(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                              size_t ws_bytes, void* stream, int32_t* d_out, uint64_t cap, uint64_t* n_total,
                              tdfs_stats* stats) {
  if (!g || !p || !n_total) return fail(TDFS_E_INVALID_ARG, "enumerate: NULL graph, plan or n_total");
  if (cap > 0 && !d_out) return fail(TDFS_E_INVALID_ARG, "enumerate: d_out NULL with cap > 0");
  tdfs_run_opts d;
  if (!o) {
    tdfs_run_opts_default(&d);
    o = &d;
  }
  return launch_job(graph_of(g), plan_of(p), o, workspace, ws_bytes, stream, 1, d_out, cap, nullptr, true, n_total,
                    stats, nullptr, 0, nullptr);
}

extern "C" int tdfs_enumerate_stream(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                                     size_t ws_bytes, void* stream, int32_t* d_ring, uint64_t ring_cap,
                                     tdfs_tuple_sink sink, void* user, uint64_t* n_total) {
  if (!g || !p) return fail(TDFS_E_INVALID_ARG, "enumerate_stream: NULL graph or plan");
  tdfs_run_opts d;
  if (!o) {
    tdfs_run_opts_default(&d);
    o = &d;
  }
  return stream_job(graph_of(g), plan_of(p), o, workspace, ws_bytes, stream, d_ring, ring_cap, sink, user, n_total);
}

namespace {
struct FileSink {
  FILE* f;
  bool bad;
};
int file_sink(const int32_t* t, uint64_t n, int32_t k, void* user) {
  FileSink* s = static_cast<FileSink*>(user);
  if (std::fwrite(t, sizeof(int32_t) * (size_t)k, (size_t)n, s->f) != (size_t)n) {
    s->bad = true;
    return 1;
  }
  return 0;
}
}  // namespace

extern "C" int tdfs_enumerate_to_file(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                                      size_t ws_bytes, void* stream, int32_t* d_ring, uint64_t ring_cap,
                                      const char* path, uint64_t* n_total) {
  if (!path) return fail(TDFS_E_INVALID_ARG, "enumerate_to_file: NULL path");
  FileSink s{std::fopen(path, "wb"), false};
  if (!s.f) return fail(TDFS_E_INVALID_ARG, std::string("enumerate_to_file: cannot open ") + path);
  int rc = tdfs_enumerate_stream(g, p, o, workspace, ws_bytes, stream, d_ring, ring_cap, file_sink, &s, n_total);
  if (std::fclose(s.f) != 0 && rc == TDFS_OK) rc = fail(TDFS_E_INVALID_ARG, "enumerate_to_file: write failed");
  if (s.bad) rc = fail(TDFS_E_INVALID_ARG, std::string("enumerate_to_file: write failed: ") + path);
  return rc;
}

extern "C" int tdfs_workspace_status(const void* workspace, void* stream) {
  if (!workspace) return fail(TDFS_E_INVALID_ARG, "workspace_status: NULL");
  unsigned long long err = 0;
  cudaError_t e = cudaMemcpyAsync(&err, (const char*)workspace + sizeof(unsigned long long) * C_ERROR * kCounterStride,
                                  sizeof(err), cudaMemcpyDeviceToHost, (cudaStream_t)stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize((cudaStream_t)stream);
  if (e != cudaSuccess) return fail(TDFS_E_CUDA, std::string("workspace_status: ") + cudaGetErrorString(e));
  if (err) return fail(TDFS_E_STACK_EXHAUSTED, "last job exhausted the stack page pool / page table");
  return TDFS_OK;
}

extern "C" int tdfs_test_count_trace(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                                     size_t ws_bytes, void* stream, int32_t* h_trace, int64_t cap, int64_t* n_trace,
                                     uint64_t* h_count) {
  if (!g || !p || !h_trace || cap <= 0 || !n_trace || !h_count) return fail(TDFS_E_INVALID_ARG, "count_trace: bad args");
  tdfs_run_opts d;
  if (!o) {
    tdfs_run_opts_default(&d);
    o = &d;
  }
  return launch_job(graph_of(g), plan_of(p), o, workspace, ws_bytes, stream, 0, nullptr, 0, nullptr, true, h_count,
                    nullptr, h_trace, cap, n_trace);
}
