// Host-buffer driver of the hot path (vpic_run_host, include/vpic.h): whole
// sort periods whose inputs come from, and whose result goes back to, pinned
// HOST memory, the copies pipelined under the neighbouring periods' compute.
// It strings together the same C-ABI calls a caller would (sort, load
// interpolator, clear, advance_p per species, [migrate], unload, [field
// solve]) -- one entry point through which the end-to-end number of bench.py
// is measured.
//
// Buffers (per species, caller device memory): four particle buffers rotate
// through "input of this period" / "sort output" / "upload of the next
// period" / "download of the previous period".  Streams: the caller's stream
// computes; two internal non-blocking streams copy host->device and
// device->host, ordered against the compute with events:
//   period k+1's upload (H2D)  ||  period k's compute  ||  period k-1's download (D2H).
#include <cstring>
#include <deque>
#include <map>
#include <utility>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "vpic_internal.cuh"

namespace {

struct Carve {
  char *base;
  size_t off, cap;
  template <class T>
  T *take(size_t bytes) {
    const size_t o = (off + 255) & ~size_t(255);
    if (o + bytes > cap) return nullptr;
    off = o + bytes;
    return reinterpret_cast<T *>(base + o);
  }
};

// workspace layout (device): fields x 2, interp, acc, jf, jf staging x 2,
// per species movers / count / flags, sort workspace
struct HostWs {
  float *fields[2], *interp, *acc, *jf, *jstage[2];
  std::vector<vpic_mover_t *> movers;
  std::vector<int64_t *> n_movers;
  std::vector<int32_t *> flags;
  void *sort_ws;
  size_t sort_ws_bytes;
  int64_t max_movers;
};

int64_t movers_cap(int64_t max_np) { return std::max<int64_t>(max_np / 8, 4096); }

bool carve(const vpic_ctx *c, int nsp, const vpic_species_host_t *sp, int order, void *ws,
           size_t ws_bytes, HostWs &w, size_t *total) {
  Carve cv{static_cast<char *>(ws), 0, ws ? ws_bytes : ~size_t(0) >> 1};
  const size_t nv = (size_t)c->gk.nv;
  bool ok = true;
  auto take = [&](auto *&ptr, size_t bytes) {
    using T = std::remove_reference_t<decltype(*ptr)>;
    ptr = cv.take<T>(bytes);
    ok = ok && ptr != nullptr;
  };
  for (int k = 0; k < 2; ++k) take(w.fields[k], nv * 32);
  take(w.interp, nv * 96);
  take(w.acc, nv * 48);
  take(w.jf, nv * 16);
  for (int k = 0; k < 2; ++k) take(w.jstage[k], nv * 16);
  int64_t max_np = 0;
  for (int j = 0; j < nsp; ++j) max_np = std::max(max_np, sp[j].max_np);
  w.max_movers = movers_cap(max_np);
  w.movers.assign(nsp, nullptr);
  w.n_movers.assign(nsp, nullptr);
  w.flags.assign(nsp, nullptr);
  for (int j = 0; j < nsp; ++j) {
    take(w.movers[j], (size_t)w.max_movers * 16);
    take(w.n_movers[j], 8);
    take(w.flags[j], 4);
  }
  w.sort_ws_bytes = order == VPIC_SORT_NONE ? 0 : vpic::sort_workspace_bytes(c, max_np, order);
  w.sort_ws = w.sort_ws_bytes ? cv.take<char>(w.sort_ws_bytes) : nullptr;
  ok = ok && (w.sort_ws_bytes == 0 || w.sort_ws != nullptr);
  if (total) *total = cv.off + 256;
  return ok;
}

}  // namespace

extern "C" {

size_t vpic_run_host_workspace_bytes(const vpic_ctx *c, int nsp, const vpic_species_host_t *sp,
                                     int order) {
  if (!c || nsp < 1 || !sp || order < 0 || order > 3) return 0;
  HostWs w;
  size_t total = 0;
  carve(c, nsp, sp, order, nullptr, 0, w, &total);
  return total;
}

int vpic_run_host(vpic_ctx *c, int nsp, const vpic_species_host_t *sp, const float *fields_host,
                  float *jf_host, int order, int64_t tile_sz, int steps, int n_cycles,
                  const int8_t *deposit_modes, int field_solve, float eps0, void *ws, size_t ws_bytes,
                  int64_t *pushes, void *stream) {
  if (!c || nsp < 1 || nsp > 16 || !sp || !fields_host || !jf_host || order < 0 || order > 3 ||
      steps < 1 || n_cycles < 1 || !ws || (field_solve && !(eps0 > 0)))
    return VPIC_ERR_INVALID;
  for (int j = 0; j < nsp; ++j) {
    if (!sp[j].host_in || sp[j].np < 0 || sp[j].np > sp[j].max_np || !(sp[j].m > 0)) return VPIC_ERR_INVALID;
    for (int b = 0; b < 4; ++b)
      if (!sp[j].dev[b] || (reinterpret_cast<uintptr_t>(sp[j].dev[b]) & 15u)) return VPIC_ERR_INVALID;
  }
  if (deposit_modes)
    for (int k = 0; k < steps * nsp; ++k)
      if (deposit_modes[k] < vpic::DEP_AUTO || deposit_modes[k] > vpic::DEP_SMEM) return VPIC_ERR_INVALID;
  HostWs w;
  size_t need = 0;
  if (!carve(c, nsp, sp, order, ws, ws_bytes, w, &need) || ws_bytes < need) return VPIC_ERR_CAPACITY;
  nvtxRangePushA(__func__);
  int dev_prev = -1;
  if (cudaGetDevice(&dev_prev) != cudaSuccess) dev_prev = -1;
  if (dev_prev != c->device) cudaSetDevice(c->device);

  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const size_t nv = (size_t)c->gk.nv;
  const bool migrate = c->ex != nullptr || [&] {
    for (int f = 0; f < 6; ++f)
      if (c->gk.face_kind[f] == vpic::FACE_ABSORB) return true;
    return false;
  }();
  const int dep0 = c->deposit;
  cudaStream_t h2d = nullptr, d2h = nullptr;
  std::vector<cudaEvent_t> events;
  int rc = VPIC_OK;
  auto ev_new = [&]() {
    cudaEvent_t e = nullptr;
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return (cudaEvent_t) nullptr;
    events.push_back(e);
    return e;
  };
#define RH_CK(x) do { if ((x) != cudaSuccess) { rc = VPIC_ERR_CUDA; goto done; } } while (0)
#define RH_RC(x) do { const int r_ = (x); if (r_ != VPIC_OK) { rc = r_; goto done; } } while (0)
  {
    RH_CK(cudaStreamCreateWithFlags(&h2d, cudaStreamNonBlocking));
    RH_CK(cudaStreamCreateWithFlags(&d2h, cudaStreamNonBlocking));
    std::vector<int> IN(nsp, 0), SC(nsp, 1);
    std::vector<std::deque<int>> SPARE(nsp, std::deque<int>{2, 3});
    std::map<std::pair<int, int>, cudaEvent_t> free_ev;    // (species, buffer) -> reusable after
    std::vector<cudaEvent_t> ev_comp(n_cycles, nullptr), ev_out(n_cycles, nullptr);
    std::vector<int64_t> np(nsp);
    int64_t total = 0;
    auto upload = [&](int k, const std::vector<int> &bufs) -> cudaEvent_t {
      for (int j = 0; j < nsp; ++j) {
        auto it = free_ev.find({j, bufs[j]});
        if (it != free_ev.end()) {
          if (cudaStreamWaitEvent(h2d, it->second, 0) != cudaSuccess) return nullptr;
          free_ev.erase(it);
        }
        if (sp[j].np && cudaMemcpyAsync(sp[j].dev[bufs[j]], sp[j].host_in, 32 * (size_t)sp[j].np,
                                        cudaMemcpyHostToDevice, h2d) != cudaSuccess)
          return nullptr;
      }
      if (k >= 2 && cudaStreamWaitEvent(h2d, ev_comp[k - 2], 0) != cudaSuccess) return nullptr;  // fields[k%2]
      if (cudaMemcpyAsync(w.fields[k % 2], fields_host, nv * 32, cudaMemcpyHostToDevice, h2d) != cudaSuccess)
        return nullptr;
      cudaEvent_t e = ev_new();
      if (!e || cudaEventRecord(e, h2d) != cudaSuccess) return nullptr;
      return e;
    };
    cudaEvent_t ev_in = upload(0, IN);
    if (!ev_in) { rc = VPIC_ERR_CUDA; goto done; }
    for (int k = 0; k < n_cycles; ++k) {
      std::vector<int> nxt;
      cudaEvent_t ev_next = nullptr;
      if (k + 1 < n_cycles) {
        for (int j = 0; j < nsp; ++j) { nxt.push_back(SPARE[j].front()); SPARE[j].pop_front(); }
        ev_next = upload(k + 1, nxt);
        if (!ev_next) { rc = VPIC_ERR_CUDA; goto done; }
      }
      RH_CK(cudaStreamWaitEvent(s, ev_in, 0));
      std::vector<vpic_particle_t *> cur(nsp), scr(nsp);
      for (int j = 0; j < nsp; ++j) {
        cur[j] = sp[j].dev[IN[j]];
        scr[j] = sp[j].dev[SC[j]];
        np[j] = sp[j].np;
      }
      float *fields = w.fields[k % 2];
      for (int t = 0; t < steps; ++t) {
        if (t == 0 && order != VPIC_SORT_NONE)
          for (int j = 0; j < nsp; ++j) {
            RH_RC(vpic_sort_particles(c, cur[j], scr[j], np[j], order, tile_sz, w.sort_ws, w.sort_ws_bytes,
                                      nullptr, nullptr, nullptr, s));
            std::swap(cur[j], scr[j]);
          }
        RH_RC(vpic_load_interpolator(c, fields, w.interp, s));
        RH_RC(vpic_clear_accumulator(c, w.acc, s));
        for (int j = 0; j < nsp; ++j) {
          if (deposit_modes) c->deposit = deposit_modes[t * nsp + j];
          if (migrate) RH_CK(cudaMemsetAsync(w.n_movers[j], 0, 8, s));
          RH_RC(vpic_advance_p(c, sp[j].q, sp[j].m, cur[j], np[j], w.interp, w.acc, w.movers[j], w.max_movers,
                               w.n_movers[j], w.flags[j], s));
          if (migrate)
            RH_RC(vpic_migrate_particles(c, sp[j].q, sp[j].m, cur[j], &np[j], sp[j].max_np, w.movers[j],
                                         w.max_movers, w.n_movers[j], w.acc, s));
        }
        RH_RC(vpic_unload_accumulator(c, w.acc, w.jf, s));
        if (field_solve) {
          RH_RC(vpic_advance_b(c, fields, 0.5f, s));
          RH_RC(vpic_advance_e(c, fields, w.jf, eps0, s));
          RH_RC(vpic_advance_b(c, fields, 0.5f, s));
        }
        for (int j = 0; j < nsp; ++j) total += np[j];
      }
      if (k >= 2) RH_CK(cudaStreamWaitEvent(s, ev_out[k - 2], 0));   // jf staging buffer downloaded
      RH_CK(cudaMemcpyAsync(w.jstage[k % 2], w.jf, nv * 16, cudaMemcpyDeviceToDevice, s));
      ev_comp[k] = ev_new();
      if (!ev_comp[k]) { rc = VPIC_ERR_CUDA; goto done; }
      RH_CK(cudaEventRecord(ev_comp[k], s));
      std::vector<int> res(nsp);
      for (int j = 0; j < nsp; ++j) res[j] = cur[j] == sp[j].dev[IN[j]] ? IN[j] : SC[j];
      RH_CK(cudaStreamWaitEvent(d2h, ev_comp[k], 0));
      for (int j = 0; j < nsp; ++j)
        if (sp[j].host_out && np[j])
          RH_CK(cudaMemcpyAsync(sp[j].host_out, cur[j], 32 * (size_t)np[j], cudaMemcpyDeviceToHost, d2h));
      RH_CK(cudaMemcpyAsync(jf_host, w.jstage[k % 2], nv * 16, cudaMemcpyDeviceToHost, d2h));
      ev_out[k] = ev_new();
      if (!ev_out[k]) { rc = VPIC_ERR_CUDA; goto done; }
      RH_CK(cudaEventRecord(ev_out[k], d2h));
      for (int j = 0; j < nsp; ++j) {
        free_ev[{j, res[j]}] = ev_out[k];
        const int other = res[j] == IN[j] ? SC[j] : IN[j];
        SPARE[j].push_back(res[j]);
        if (!nxt.empty()) {
          IN[j] = nxt[j];
          SC[j] = other;
        }
      }
      ev_in = ev_next;
    }
    if (pushes) *pushes = total;
  }
done:
  c->deposit = dep0;
  // the caller's stream waits for both copy streams (its synchronisation
  // covers every copy of the call)
  for (cudaStream_t cs : {h2d, d2h}) {
    if (!cs) continue;
    cudaEvent_t e = ev_new();
    if (e && cudaEventRecord(e, cs) == cudaSuccess) cudaStreamWaitEvent(s, e, 0);
    cudaStreamDestroy(cs);   // released once its work completes
  }
  for (cudaEvent_t e : events)
    if (e) cudaEventDestroy(e);
  if (dev_prev >= 0 && dev_prev != c->device) cudaSetDevice(dev_prev);
  nvtxRangePop();
  return rc;
#undef RH_CK
#undef RH_RC
}

}  // extern "C"
