// versioned.cu — searches concurrent with bulk updates (the
// paper's concurrent search / update experiment, App. B.3, and its
// batch update, §5.6).
//
// The paper serialises concurrent queries with per-node mutexes on the CPU copy and
// re-synchronises the GPU I-segment after the batch.  On B200 the whole tree is
// device-resident, so the B200 form is multi-versioning: a versioned handle owns a
// sequence of immutable tree versions.
//   hbt_versioned_search  reads the version current at the call, on the caller's
//                         stream, and records a CUDA event after its kernels;
//   hbt_versioned_update  builds version k+1 from version k on ITS stream —
//                         implicit: merge + rebuild into fresh arrays;
//                         regular: a device-to-device copy of version k, then the
//                         in-place batch update (R11) on the copy — while searches
//                         on other streams keep reading version k; then publishes
//                         k+1 under the handle's mutex (host-side pointer swap);
//   retirement            a replaced version is freed once no host call is inside
//                         it and every event its searches recorded has completed.
// Every search therefore returns exactly the result of the version it started on
// (tests/test_gpu_concurrency.py checks this against the oracle per version).
#include <vector>

#include "hbt_internal.cuh"

namespace hbt {
namespace {

struct Version {
  hbt_tree* t = nullptr;
  uint64_t ver = 0;
  int active = 0;                   // host calls currently launching on this version
  std::vector<cudaEvent_t> events;  // completion of the searches launched on it
};

}  // namespace
}  // namespace hbt

struct hbt_versioned {
  std::mutex mu;         // the version list
  std::mutex update_mu;  // one update at a time
  std::vector<hbt::Version> vs;  // vs.back() is current
};

namespace hbt {
namespace {

// Free retired versions whose searches are done (caller holds v->mu).
void collect(hbt_versioned* v) {
  for (size_t i = 0; i + 1 < v->vs.size();) {
    Version& x = v->vs[i];
    bool done = x.active == 0;
    for (size_t e = 0; done && e < x.events.size(); ++e) {
      const cudaError_t q = cudaEventQuery(x.events[e]);
      if (q == cudaErrorNotReady) done = false;
      else if (q != cudaSuccess) cudaGetLastError();  // a failed search: nothing left to wait for
    }
    if (!done) { ++i; continue; }
    for (cudaEvent_t e : x.events) cudaEventDestroy(e);
    free_tree(x.t);
    v->vs.erase(v->vs.begin() + long(i));
  }
  // searches on the current version keep appending events: drop the completed ones
  Version& c = v->vs.back();
  size_t w = 0;
  for (size_t e = 0; e < c.events.size(); ++e) {
    if (cudaEventQuery(c.events[e]) == cudaErrorNotReady) c.events[w++] = c.events[e];
    else { cudaGetLastError(); cudaEventDestroy(c.events[e]); }
  }
  c.events.resize(w);
}

Version* find(hbt_versioned* v, hbt_tree* t) {
  for (Version& x : v->vs)
    if (x.t == t) return &x;
  return nullptr;
}

// An empty tree object with src's parameters and launch configuration.
hbt_tree* empty_like(const hbt_tree* src) {
  hbt_tree* t = new hbt_tree();
  t->form = src->form;
  t->width = src->width;
  t->F = src->F;
  t->P = src->P;
  t->device = src->device;
  t->num_sms = src->num_sms;
  t->cfg = src->cfg;
  return t;
}

}  // namespace
}  // namespace hbt

using namespace hbt;

extern "C" {

int hbt_versioned_create(hbt_tree* t, hbt_versioned** out) {
  if (!t || !out) { set_error("NULL argument"); return HBT_EINVAL; }
  *out = nullptr;
  if (t->shard.G >= 1) { set_error("versioned trees are not key-range shards"); return HBT_EUNSUPPORTED; }
  if (t->h_leaf || t->r.h_leaf) { set_error("versioned trees keep their L-segment in HBM"); return HBT_EUNSUPPORTED; }
  hbt_versioned* v = new hbt_versioned();
  Version x;
  x.t = t;
  x.ver = 0;
  v->vs.push_back(x);
  *out = v;
  return HBT_OK;
}

int hbt_versioned_search(hbt_versioned* v, const void* queries, uint64_t m, hbt_out out, void* stream,
                         uint64_t* version) {
  if (!v) { set_error("NULL handle"); return HBT_EINVAL; }
  NvtxRange nvtx_("hbt_versioned_search");
  hbt_tree* t;
  {
    std::lock_guard<std::mutex> lock(v->mu);
    Version& c = v->vs.back();
    ++c.active;
    t = c.t;
    if (version) *version = c.ver;
  }
  int rc = hbt_search(t, queries, m, out, stream);
  cudaEvent_t ev = nullptr;
  cudaError_t e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventRecord(ev, (cudaStream_t)stream);
  std::lock_guard<std::mutex> lock(v->mu);
  Version* x = find(v, t);
  --x->active;
  if (e == cudaSuccess) {
    x->events.push_back(ev);
  } else {
    // no event: wait for the stream instead, so the version cannot be freed under it
    cudaGetLastError();
    if (ev) cudaEventDestroy(ev);
    cudaStreamSynchronize((cudaStream_t)stream);
    if (rc == HBT_OK) { set_error("search completion event: %s", cudaGetErrorString(e)); rc = HBT_ECUDA; }
  }
  collect(v);
  return rc;
}

int hbt_versioned_update(hbt_versioned* v, const hbt_batch* batch, void* stream, uint64_t* version) {
  if (!v || !batch) { set_error("NULL argument"); return HBT_EINVAL; }
  NvtxRange nvtx_("hbt_versioned_update");
  std::lock_guard<std::mutex> ulock(v->update_mu);
  cudaStream_t s = (cudaStream_t)stream;
  hbt_tree* base;
  uint64_t bver;
  {
    std::lock_guard<std::mutex> lock(v->mu);
    Version& c = v->vs.back();
    ++c.active;  // the base stays alive while version k+1 is derived from it
    base = c.t;
    bver = c.ver;
  }
  auto release = [&]() {
    std::lock_guard<std::mutex> lock(v->mu);
    --find(v, base)->active;
    collect(v);
  };
  if (batch->count == 0) {
    release();
    if (version) *version = bver;
    return HBT_OK;
  }
  hbt_tree* nt = empty_like(base);
  int rc;
  if (base->form == HBT_IMPLICIT) {
    rc = implicit_merge_rebuild(base, batch, nt, s);
  } else {
    nt->n = base->n;
    rc = regular_clone(base, nt, s);
    if (rc == HBT_OK) rc = hbt_bulk_update(nt, batch, stream);
  }
  if (rc != HBT_OK) {
    free_tree(nt);
    release();
    return rc;
  }
  {
    std::lock_guard<std::mutex> lock(v->mu);
    Version x;
    x.t = nt;
    x.ver = bver + 1;
    v->vs.push_back(x);
    --find(v, base)->active;
    if (version) *version = x.ver;
    collect(v);
  }
  return HBT_OK;
}

int hbt_versioned_current(hbt_versioned* v, hbt_tree** t, uint64_t* version) {
  if (!v || !t) { set_error("NULL argument"); return HBT_EINVAL; }
  std::lock_guard<std::mutex> lock(v->mu);
  *t = v->vs.back().t;
  if (version) *version = v->vs.back().ver;
  return HBT_OK;
}

int hbt_versioned_destroy(hbt_versioned* v) {
  if (!v) return HBT_EINVAL;
  cudaDeviceSynchronize();
  for (Version& x : v->vs) {
    for (cudaEvent_t e : x.events) cudaEventDestroy(e);
    free_tree(x.t);
  }
  delete v;
  return HBT_OK;
}

}  // extern "C"
