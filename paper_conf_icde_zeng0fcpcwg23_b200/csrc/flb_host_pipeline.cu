// flb_host_pipeline.cu — host-buffer entry points (PAPER Fig. 4, §V-A).
//
// The paper's pipeline moves host data through "data processing / compression -> copy to GPU ->
// GPU HE -> copy back" (encryption ①–④, decryption ⑤–⑨, homomorphic computation ④⑤).  These
// calls take HOST buffers, split the batch into chunks and run chunk i's H2D copy, kernels and
// D2H copy on one of two internal streams while the host copies chunk i-1 out of pinned staging
// memory, so transfers overlap the (dominant) HE kernels.  They are built only on the public
// batch entry points of flb_paillier.h (layer L3 over L1/L2) and return when the host output is
// complete.  Pinned staging and device buffers are per device, grown on demand and reused; a caller
// buffer that is itself page-locked (cudaHostAlloc / cudaHostRegister, e.g. a pin_memory tensor) is
// copied from / into directly, without the staging memcpy.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <map>
#include <mutex>
#include <string>

#include "../../include/flb_paillier.h"

namespace flb {
void set_last_error(const std::string& msg);  // flb_api.cu: the message flb_last_error() returns
void set_half_units(bool on);                 // flb_api.cu: half units for incomplete last rounds
}

namespace {

struct ErrSink {
  ErrSink& operator=(const std::string& m) {
    flb::set_last_error(m);
    return *this;
  }
};
thread_local ErrSink g_perr;

struct Buf {
  void* p = nullptr;
  size_t cap = 0;
};

struct DevCtx {
  std::mutex mu;
  cudaStream_t st[2] = {nullptr, nullptr};
  cudaEvent_t done[2] = {nullptr, nullptr};
  Buf pin_in[2], pin_out[2], pin_aux[2];
  Buf d_in[2], d_mid[2], d_out[2], d_aux[2];
};

#define PCK(call)                                                              \
  do {                                                                         \
    cudaError_t e_ = (call);                                                   \
    if (e_ != cudaSuccess) {                                                   \
      g_perr = std::string(#call) + ": " + cudaGetErrorString(e_);             \
      return FLB_ECUDA;                                                        \
    }                                                                          \
  } while (0)

int ctx_for_device(DevCtx** out) {
  static std::mutex mu;
  static std::map<int, DevCtx*> ctxs;
  int dev;
  PCK(cudaGetDevice(&dev));
  std::lock_guard<std::mutex> lk(mu);
  DevCtx*& c = ctxs[dev];
  if (!c) {
    c = new DevCtx();
    for (int i = 0; i < 2; i++) {
      PCK(cudaStreamCreateWithFlags(&c->st[i], cudaStreamNonBlocking));
      PCK(cudaEventCreateWithFlags(&c->done[i], cudaEventDisableTiming));
    }
  }
  *out = c;
  return FLB_OK;
}

int ensure_host(Buf& b, size_t need) {
  if (b.cap >= need) return FLB_OK;
  if (b.p) PCK(cudaFreeHost(b.p));
  b.p = nullptr;
  b.cap = 0;
  PCK(cudaHostAlloc(&b.p, need, cudaHostAllocDefault));
  b.cap = need;
  return FLB_OK;
}

int ensure_dev(Buf& b, size_t need) {
  if (b.cap >= need) return FLB_OK;
  if (b.p) PCK(cudaFree(b.p));
  b.p = nullptr;
  b.cap = 0;
  PCK(cudaMalloc(&b.p, need));
  b.cap = need;
  return FLB_OK;
}

int lib_err(int rc, const char* what) {
  g_perr = std::string(what) + ": " + flb_last_error();  // prefix the entry point that failed
  return rc;
}

#define RC(x)                 \
  do {                        \
    int rc_ = (x);            \
    if (rc_) return rc_;      \
  } while (0)

constexpr size_t kChunkPt = 32768;  // plaintexts / ciphertexts per pipeline chunk (at most)

// Equal chunks of at most kChunkPt rows (multiples of the 128-element tensor-core tile): a batch of
// 4 kChunkPt + a few rows would otherwise end in a tiny launch that runs on a nearly idle GPU.
size_t chunk_rows(size_t total) {
  const size_t chunks = (total + kChunkPt - 1) / kChunkPt;
  if (chunks <= 1) return total ? total : 1;
  const size_t c = (total + chunks - 1) / chunks;
  return std::min(kChunkPt, (c + 127) / 128 * 128);
}

// [p, p + bytes) lies in page-locked host memory (cudaHostAlloc / cudaHostRegister): the copies DMA
// straight from / into the caller's buffer, no staging memcpy
bool is_pinned(const void* p, size_t bytes) {
  auto one = [](const void* q) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, q) != cudaSuccess) {
      (void)cudaGetLastError();
      return false;
    }
    return a.type == cudaMemoryTypeHost;
  };
  return p && bytes && one(p) && one((const char*)p + bytes - 1);
}

}  // namespace

extern "C" {

int flb_pack_encrypt_host(const flb_pub* pub, const flb_priv* priv, const flb_codec* codec, const float* x_host,
                          size_t n_values, uint64_t seed, uint64_t ctr0, uint32_t* c_host) {
  if (!pub || !codec || !x_host || !c_host || codec->slots == 0) {
    g_perr = "null pointer or zero slots";
    return FLB_EINVAL;
  }
  if (n_values == 0) return FLB_OK;
  DevCtx* C;
  RC(ctx_for_device(&C));
  std::lock_guard<std::mutex> lk(C->mu);
  const size_t S = codec->slots, ptw = flb_pt_words(pub), ctw = flb_ct_words(pub);
  const size_t n_pt = (n_values + S - 1) / S;
  const size_t rows = chunk_rows(n_pt), chunks = (n_pt + rows - 1) / rows;
  const bool in_pinned = is_pinned(x_host, n_values * 4), out_pinned = is_pinned(c_host, n_pt * ctw * 4);
  for (int s = 0; s < 2; s++) {
    RC(ensure_host(C->pin_in[s], kChunkPt * S * 4));
    RC(ensure_host(C->pin_out[s], kChunkPt * ctw * 4));
    RC(ensure_dev(C->d_in[s], kChunkPt * S * 4));
    RC(ensure_dev(C->d_mid[s], kChunkPt * ptw * 4));
    RC(ensure_dev(C->d_out[s], kChunkPt * ctw * 4));
  }
  size_t pending_pt0 = 0, pending_n = 0;
  int pending_s = -1;
  for (size_t i = 0; i < chunks; i++) {
    const int s = (int)(i & 1);
    const size_t pt0 = i * rows, npt = std::min(rows, n_pt - pt0);
    const size_t v0 = pt0 * S, nv = std::min(npt * S, n_values - v0);
    if (!in_pinned) std::memcpy(C->pin_in[s].p, x_host + v0, nv * 4);
    PCK(cudaMemcpyAsync(C->d_in[s].p, in_pinned ? (const void*)(x_host + v0) : C->pin_in[s].p, nv * 4,
                        cudaMemcpyHostToDevice, C->st[s]));
    int rc = flb_pack(pub, codec, (const float*)C->d_in[s].p, nv, (uint32_t*)C->d_mid[s].p, C->st[s]);
    if (rc) return lib_err(rc, "flb_pack");
    rc = priv ? flb_encrypt_crt(priv, (const uint32_t*)C->d_mid[s].p, nullptr, seed, ctr0 + pt0,
                                (uint32_t*)C->d_out[s].p, npt, C->st[s])
              : flb_encrypt(pub, (const uint32_t*)C->d_mid[s].p, nullptr, seed, ctr0 + pt0,
                            (uint32_t*)C->d_out[s].p, npt, C->st[s]);
    if (rc) return lib_err(rc, "flb_encrypt");
    PCK(cudaMemcpyAsync(out_pinned ? (void*)(c_host + pt0 * ctw) : C->pin_out[s].p, C->d_out[s].p, npt * ctw * 4,
                        cudaMemcpyDeviceToHost, C->st[s]));
    PCK(cudaEventRecord(C->done[s], C->st[s]));
    if (pending_s >= 0) {  // drain the previous chunk while this one runs
      PCK(cudaEventSynchronize(C->done[pending_s]));
      if (!out_pinned) std::memcpy(c_host + pending_pt0 * ctw, C->pin_out[pending_s].p, pending_n * ctw * 4);
    }
    pending_s = s;
    pending_pt0 = pt0;
    pending_n = npt;
  }
  PCK(cudaEventSynchronize(C->done[pending_s]));
  if (!out_pinned) std::memcpy(c_host + pending_pt0 * ctw, C->pin_out[pending_s].p, pending_n * ctw * 4);
  return FLB_OK;
}

int flb_pack_encrypt_host_multi(const flb_pub* pub, const flb_priv* priv, const flb_codec* codec,
                                const float* const* x_hosts, const size_t* n_values, size_t n_arrays, uint64_t seed,
                                uint64_t ctr0, uint32_t* c_host) {
  if (!pub || !codec || !x_hosts || !n_values || !c_host || codec->slots == 0) {
    g_perr = "null pointer or zero slots";
    return FLB_EINVAL;
  }
  if (n_arrays == 0) return FLB_OK;
  DevCtx* C;
  RC(ctx_for_device(&C));
  std::lock_guard<std::mutex> lk(C->mu);
  const size_t S = codec->slots, ptw = flb_pt_words(pub), ctw = flb_ct_words(pub);
  size_t total_v = 0, total_pt = 0;
  for (size_t a = 0; a < n_arrays; a++) {
    if (n_values[a] && !x_hosts[a]) {
      g_perr = "null array";
      return FLB_EINVAL;
    }
    total_v += n_values[a];
    total_pt += (n_values[a] + S - 1) / S;
  }
  if (total_pt == 0) return FLB_OK;
  // all values in (pinned staging, one H2D per array on stream 0), every array packed into its own
  // plaintexts (slot alignment per array), then encryption in chunks with D2H overlap on 2 streams
  RC(ensure_host(C->pin_aux[0], total_v * 4 + 16));
  RC(ensure_dev(C->d_aux[0], total_v * 4 + 16));
  RC(ensure_dev(C->d_mid[0], total_pt * ptw * 4));
  for (int s = 0; s < 2; s++) {
    RC(ensure_host(C->pin_out[s], kChunkPt * ctw * 4));
    RC(ensure_dev(C->d_out[s], kChunkPt * ctw * 4));
  }
  size_t v0 = 0, p0 = 0;
  for (size_t a = 0; a < n_arrays; a++) {
    if (!n_values[a]) continue;
    const float* src = x_hosts[a];
    if (!is_pinned(src, n_values[a] * 4)) {
      std::memcpy((float*)C->pin_aux[0].p + v0, x_hosts[a], n_values[a] * 4);
      src = (const float*)C->pin_aux[0].p + v0;
    }
    PCK(cudaMemcpyAsync((float*)C->d_aux[0].p + v0, src, n_values[a] * 4, cudaMemcpyHostToDevice, C->st[0]));
    int rc = flb_pack(pub, codec, (const float*)C->d_aux[0].p + v0, n_values[a], (uint32_t*)C->d_mid[0].p + p0 * ptw,
                      C->st[0]);
    if (rc) return lib_err(rc, "flb_pack");
    v0 += n_values[a];
    p0 += (n_values[a] + S - 1) / S;
  }
  PCK(cudaEventRecord(C->done[0], C->st[0]));
  PCK(cudaStreamWaitEvent(C->st[1], C->done[0], 0));
  // Equal chunks on two streams: chunk i+1's CTAs fill chunk i's last round, so only the final chunk
  // ends its last round with half units (flb_tc.cuh); D2H of chunk i overlaps chunk i+1.
  const bool out_pinned = is_pinned(c_host, total_pt * ctw * 4);
  const size_t rows = chunk_rows(total_pt), chunks = (total_pt + rows - 1) / rows;
  struct HalfUnits {
    ~HalfUnits() { flb::set_half_units(true); }
  } restore;
  size_t pending_pt0 = 0, pending_n = 0;
  int pending_s = -1;
  for (size_t i = 0; i < chunks; i++) {
    const int s = (int)(i & 1);
    const size_t pt0 = i * rows, npt = std::min(rows, total_pt - pt0);
    const uint32_t* src = (const uint32_t*)C->d_mid[0].p + pt0 * ptw;
    flb::set_half_units(i + 1 == chunks);
    int rc = priv ? flb_encrypt_crt(priv, src, nullptr, seed, ctr0 + pt0, (uint32_t*)C->d_out[s].p, npt, C->st[s])
                  : flb_encrypt(pub, src, nullptr, seed, ctr0 + pt0, (uint32_t*)C->d_out[s].p, npt, C->st[s]);
    if (rc) return lib_err(rc, "flb_encrypt");
    PCK(cudaMemcpyAsync(out_pinned ? (void*)(c_host + pt0 * ctw) : C->pin_out[s].p, C->d_out[s].p, npt * ctw * 4,
                        cudaMemcpyDeviceToHost, C->st[s]));
    PCK(cudaEventRecord(C->done[s], C->st[s]));
    if (pending_s >= 0) {
      PCK(cudaEventSynchronize(C->done[pending_s]));  // (d_out[s] and pin_out[s] are free again)
      if (!out_pinned) std::memcpy(c_host + pending_pt0 * ctw, C->pin_out[pending_s].p, pending_n * ctw * 4);
    }
    pending_s = s;
    pending_pt0 = pt0;
    pending_n = npt;
  }
  PCK(cudaEventSynchronize(C->done[pending_s]));
  if (pending_s == 1) PCK(cudaEventSynchronize(C->done[0]));
  if (!out_pinned) std::memcpy(c_host + pending_pt0 * ctw, C->pin_out[pending_s].p, pending_n * ctw * 4);
  return FLB_OK;
}

int flb_decrypt_unpack_host(const flb_priv* priv, const flb_pub* pub, const flb_codec* codec,
                            const uint32_t* c_host, size_t n_values, const uint32_t* summands_host,
                            uint32_t summands_scalar, float* x_host) {
  if (!priv || !pub || !codec || !c_host || !x_host || codec->slots == 0) {
    g_perr = "null pointer or zero slots";
    return FLB_EINVAL;
  }
  if (n_values == 0) return FLB_OK;
  DevCtx* C;
  RC(ctx_for_device(&C));
  std::lock_guard<std::mutex> lk(C->mu);
  const size_t S = codec->slots, ptw = flb_pt_words(pub), ctw = flb_ct_words(pub);
  const size_t n_ct = (n_values + S - 1) / S;
  const size_t rows = chunk_rows(n_ct), chunks = (n_ct + rows - 1) / rows;
  const bool in_pinned = is_pinned(c_host, n_ct * ctw * 4), out_pinned = is_pinned(x_host, n_values * 4);
  for (int s = 0; s < 2; s++) {
    RC(ensure_host(C->pin_in[s], kChunkPt * ctw * 4));
    RC(ensure_host(C->pin_out[s], kChunkPt * S * 4));
    RC(ensure_host(C->pin_aux[s], kChunkPt * 4));
    RC(ensure_dev(C->d_in[s], kChunkPt * ctw * 4));
    RC(ensure_dev(C->d_mid[s], kChunkPt * ptw * 4));
    RC(ensure_dev(C->d_out[s], kChunkPt * S * 4));
    RC(ensure_dev(C->d_aux[s], kChunkPt * 4));
  }
  size_t pending_v0 = 0, pending_nv = 0;
  int pending_s = -1;
  for (size_t i = 0; i < chunks; i++) {
    const int s = (int)(i & 1);
    const size_t c0 = i * rows, nc = std::min(rows, n_ct - c0);
    const size_t v0 = c0 * S, nv = std::min(nc * S, n_values - v0);
    if (!in_pinned) std::memcpy(C->pin_in[s].p, c_host + c0 * ctw, nc * ctw * 4);
    PCK(cudaMemcpyAsync(C->d_in[s].p, in_pinned ? (const void*)(c_host + c0 * ctw) : C->pin_in[s].p, nc * ctw * 4,
                        cudaMemcpyHostToDevice, C->st[s]));
    const uint32_t* dsum = nullptr;
    if (summands_host) {
      std::memcpy(C->pin_aux[s].p, summands_host + c0, nc * 4);
      PCK(cudaMemcpyAsync(C->d_aux[s].p, C->pin_aux[s].p, nc * 4, cudaMemcpyHostToDevice, C->st[s]));
      dsum = (const uint32_t*)C->d_aux[s].p;
    }
    int rc = flb_decrypt(priv, (const uint32_t*)C->d_in[s].p, (uint32_t*)C->d_mid[s].p, nc, C->st[s]);
    if (rc) return lib_err(rc, "flb_decrypt");
    rc = flb_unpack(pub, codec, (const uint32_t*)C->d_mid[s].p, nv, dsum, summands_scalar, (float*)C->d_out[s].p,
                    C->st[s]);
    if (rc) return lib_err(rc, "flb_unpack");
    PCK(cudaMemcpyAsync(out_pinned ? (void*)(x_host + v0) : C->pin_out[s].p, C->d_out[s].p, nv * 4,
                        cudaMemcpyDeviceToHost, C->st[s]));
    PCK(cudaEventRecord(C->done[s], C->st[s]));
    if (pending_s >= 0) {
      PCK(cudaEventSynchronize(C->done[pending_s]));
      if (!out_pinned) std::memcpy(x_host + pending_v0, C->pin_out[pending_s].p, pending_nv * 4);
    }
    pending_s = s;
    pending_v0 = v0;
    pending_nv = nv;
  }
  PCK(cudaEventSynchronize(C->done[pending_s]));
  if (!out_pinned) std::memcpy(x_host + pending_v0, C->pin_out[pending_s].p, pending_nv * 4);
  return FLB_OK;
}

int flb_reduce_segments_host(const flb_pub* pub, const uint32_t* c_host, size_t num_inputs, const int64_t* idx_host,
                             const int64_t* offsets_host, size_t num_segments, size_t max_segment_len,
                             uint32_t* out_host) {
  if (!pub || !offsets_host || !out_host || (num_inputs && !c_host)) {
    g_perr = "null pointer";
    return FLB_EINVAL;
  }
  if (num_segments == 0) return FLB_OK;
  DevCtx* C;
  RC(ctx_for_device(&C));
  std::lock_guard<std::mutex> lk(C->mu);
  const size_t ctw = flb_ct_words(pub);
  const size_t nidx = idx_host ? (size_t)offsets_host[num_segments] : 0;
  // inputs stream in through the two pinned staging buffers; everything else is small
  const size_t chunk = kChunkPt;
  RC(ensure_dev(C->d_in[0], std::max<size_t>(1, num_inputs) * ctw * 4));
  RC(ensure_dev(C->d_aux[0], (num_segments + 1) * 8 + nidx * 8));
  RC(ensure_dev(C->d_out[0], num_segments * ctw * 4));
  for (int s = 0; s < 2; s++) RC(ensure_host(C->pin_in[s], chunk * ctw * 4));
  RC(ensure_host(C->pin_aux[0], (num_segments + 1) * 8 + nidx * 8));
  RC(ensure_host(C->pin_out[0], num_segments * ctw * 4));
  cudaStream_t st = C->st[0];
  if (is_pinned(c_host, num_inputs * ctw * 4)) {
    PCK(cudaMemcpyAsync(C->d_in[0].p, c_host, num_inputs * ctw * 4, cudaMemcpyHostToDevice, st));
  } else {
    for (size_t c0 = 0, i = 0; c0 < num_inputs; c0 += chunk, i++) {
      const int s = (int)(i & 1);
      const size_t n = std::min(chunk, num_inputs - c0);
      if (i >= 2) PCK(cudaEventSynchronize(C->done[s]));  // staging buffer s free again
      std::memcpy(C->pin_in[s].p, c_host + c0 * ctw, n * ctw * 4);
      PCK(cudaMemcpyAsync((uint32_t*)C->d_in[0].p + c0 * ctw, C->pin_in[s].p, n * ctw * 4, cudaMemcpyHostToDevice,
                          st));
      PCK(cudaEventRecord(C->done[s], st));
    }
  }
  int64_t* aux = (int64_t*)C->pin_aux[0].p;
  std::memcpy(aux, offsets_host, (num_segments + 1) * 8);
  if (idx_host) std::memcpy(aux + num_segments + 1, idx_host, nidx * 8);
  PCK(cudaMemcpyAsync(C->d_aux[0].p, aux, (num_segments + 1 + nidx) * 8, cudaMemcpyHostToDevice, st));
  const int64_t* d_off = (const int64_t*)C->d_aux[0].p;
  const int64_t* d_idx = idx_host ? d_off + num_segments + 1 : nullptr;
  const size_t nent = idx_host ? nidx : (size_t)offsets_host[num_segments];
  int rc = flb_reduce_segments(pub, (const uint32_t*)C->d_in[0].p, num_inputs, d_idx, nent, d_off, num_segments,
                               max_segment_len, (uint32_t*)C->d_out[0].p, st);
  if (rc) return lib_err(rc, "flb_reduce_segments");
  const bool out_pinned = is_pinned(out_host, num_segments * ctw * 4);
  PCK(cudaMemcpyAsync(out_pinned ? (void*)out_host : C->pin_out[0].p, C->d_out[0].p, num_segments * ctw * 4,
                      cudaMemcpyDeviceToHost, st));
  PCK(cudaStreamSynchronize(st));
  if (!out_pinned) std::memcpy(out_host, C->pin_out[0].p, num_segments * ctw * 4);
  return FLB_OK;
}

}  // extern "C"
