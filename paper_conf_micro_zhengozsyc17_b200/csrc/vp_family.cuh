// vp_family.cuh — host-side glue between the C ABI runtime (vp_host.cu) and a workload
// family's stage functions.  A family F is a struct with:
//   static constexpr int S;                                   number of stages
//   static constexpr int kinds[S];                            vp_stage_kind per stage
//   struct Params;                                            == the vp_*_params of vp.h
//   static constexpr int stride(int s);                       item slot bytes (mult. of 4)
//   static constexpr int max_batch(int s), default_batch(int s), threads_per_item(int s);
//   static constexpr int fanout(int s, int t);                max items s emits to t per item
//   static constexpr bool uses_latches(int lo, int hi);
//   static constexpr int scratch_bytes(int lo, int hi);       extra shared memory
//   static constexpr int default_cap_log2(int s);
//   template <int s> static __device__ unsigned long long item_id(const uint8_t*);
//   template <int s, class Ctx> static __device__ void exec(Ctx&, const uint8_t* items, int n);
//   static cudaError_t init_run(const Params&, cudaStream_t);  reset sinks
//   static cudaError_t finalize(const Params&, cudaStream_t);  data-parallel resolve
//   static bool output(const Params&, int idx, void** ptr, size_t* bytes);
//   static const char* validate(const Params&);
#pragma once
#include <cuda_runtime.h>

#include "vp_runtime.cuh"

namespace vp {

struct FamilyOps {
  int S = 0;
  int kinds[kMaxStages] = {};
  const char* name = "";
  virtual ~FamilyOps() {}
  virtual int stride(int s) const = 0;
  virtual int max_batch(int s) const = 0;
  virtual int max_batch_k(int lo, int hi, bool rtc, int s) const = 0;  // per-kernel cap
  virtual int default_batch(int s) const = 0;
  virtual int threads_per_item(int s) const = 0;
  virtual int fanout(int s, int t) const = 0;
  virtual int out_cap(int lo, int hi, bool rtc, int t) const = 0;  // items a kernel publishes to t per batch
  virtual bool local_rec(int lo, int hi, bool rtc) const = 0;        // block-local recursion kernel
  virtual bool rtc_legal(int lo, int hi) const = 0;
  virtual bool latched(int lo, int hi) const = 0;
  virtual int default_cap_log2(int s) const = 0;
  virtual size_t params_bytes() const = 0;
  virtual const void* kernel(int lo, int hi, bool rtc) const = 0;
  virtual size_t smem(int lo, int hi, bool rtc) const = 0;
  virtual int block_threads(int lo, int hi, bool rtc) const = 0;  // blockDim of kernel [lo, hi]
  virtual cudaError_t launch(int lo, int hi, bool rtc, const Common& c, const GroupArgs& g, const void* params,
                             int grid, bool coop, cudaStream_t st) const = 0;
  virtual cudaError_t init_run(const void* params, cudaStream_t st) const = 0;
  virtual cudaError_t finalize(const void* params, cudaStream_t st) const = 0;
  virtual bool output(const void* params, int idx, void** ptr, size_t* bytes) const = 0;
  virtual const char* validate(const void* params) const = 0;
};

template <class F>
struct FamilyImpl final : FamilyOps {
  using G = Graph<F>;
  const void* fn[kMaxStages][kMaxStages][2] = {};
  int nthreads[kMaxStages][kMaxStages][2] = {};

  template <int LO, int HI>
  void fill() {
    if constexpr (LO < F::S) {
      if constexpr (HI < F::S) {
        fn[LO][HI][0] = (const void*)&vp_kernel<F, LO, HI, false>;
        nthreads[LO][HI][0] = Runner<F, LO, HI, false>::kBlockThreads;
        if constexpr (G::rtc_legal(LO, HI)) {
          fn[LO][HI][1] = (const void*)&vp_kernel<F, LO, HI, true>;
          nthreads[LO][HI][1] = Runner<F, LO, HI, true>::kBlockThreads;
        }
        fill<LO, HI + 1>();
      } else {
        fill<LO + 1, LO + 1>();
      }
    }
  }

  template <int LO, int HI>
  int smem_of(int lo, int hi, bool rtc) const {
    if constexpr (LO < F::S) {
      if constexpr (HI < F::S) {
        if (lo == LO && hi == HI) return G::smem_bytes(LO, HI, rtc && G::rtc_legal(LO, HI));
        return smem_of<LO, HI + 1>(lo, hi, rtc);
      } else {
        return smem_of<LO + 1, LO + 1>(lo, hi, rtc);
      }
    }
    return 0;
  }

  explicit FamilyImpl(const char* nm) {
    S = F::S;
    name = nm;
    for (int s = 0; s < F::S; ++s) kinds[s] = F::kinds[s];
    fill<0, 0>();
  }
  int stride(int s) const override { return F::stride(s); }
  int max_batch(int s) const override { return F::max_batch(s); }
  int max_batch_k(int lo, int hi, bool rtc, int s) const override { return kernel_max_batch<F>(lo, hi, rtc, s); }
  int default_batch(int s) const override { return F::default_batch(s); }
  int threads_per_item(int s) const override { return F::threads_per_item(s); }
  int fanout(int s, int t) const override { return F::fanout(s, t); }
  template <int LO, int HI>
  int out_cap_of(int lo, int hi, bool rtc, int t) const {
    if constexpr (LO < F::S) {
      if constexpr (HI < F::S) {
        if (lo == LO && hi == HI) return G::out_cap(LO, HI, rtc && G::rtc_legal(LO, HI), t);
        return out_cap_of<LO, HI + 1>(lo, hi, rtc, t);
      } else {
        return out_cap_of<LO + 1, LO + 1>(lo, hi, rtc, t);
      }
    }
    return 0;
  }
  template <int LO, int HI>
  int direct_cap_of(int lo, int hi, bool rtc, int t) const {
    if constexpr (LO < F::S) {
      if constexpr (HI < F::S) {
        if (lo == LO && hi == HI) return direct_out_cap<F>(LO, HI, rtc, t);
        return direct_cap_of<LO, HI + 1>(lo, hi, rtc, t);
      } else {
        return direct_cap_of<LO + 1, LO + 1>(lo, hi, rtc, t);
      }
    }
    return 0;
  }
  // items one block of kernel [lo, hi] can have in flight to t: its out buffer, or what
  // its warps publish at once in a direct-publish kernel
  int out_cap(int lo, int hi, bool rtc, int t) const override {
    const int d = direct_cap_of<0, 0>(lo, hi, rtc, t);
    return d > 0 ? d : out_cap_of<0, 0>(lo, hi, rtc, t);
  }
  bool local_rec(int lo, int hi, bool rtc) const override { return local_recursion<F>(lo, hi, rtc); }
  bool rtc_legal(int lo, int hi) const override { return fn[lo][hi][1] != nullptr; }
  bool latched(int lo, int hi) const override { return !F::rtc_ok(lo, hi); }
  int default_cap_log2(int s) const override { return F::default_cap_log2(s); }
  size_t params_bytes() const override { return sizeof(typename F::Params); }
  const void* kernel(int lo, int hi, bool rtc) const override { return fn[lo][hi][rtc ? 1 : 0]; }
  size_t smem(int lo, int hi, bool rtc) const override { return (size_t)smem_of<0, 0>(lo, hi, rtc); }
  int block_threads(int lo, int hi, bool rtc) const override {
    const int t = nthreads[lo][hi][rtc ? 1 : 0];
    return t > 0 ? t : kBlock;
  }
  cudaError_t launch(int lo, int hi, bool rtc, const Common& c, const GroupArgs& g, const void* params, int grid,
                     bool coop, cudaStream_t st) const override {
    const void* k = kernel(lo, hi, rtc);
    if (!k) return cudaErrorInvalidDeviceFunction;
    KArgs<F> a;
    a.c = c;
    a.g = g;
    a.p = *(const typename F::Params*)params;
    void* args[] = {&a};
    size_t sm = smem(lo, hi, rtc);
    const dim3 blk(block_threads(lo, hi, rtc));
    if constexpr (HasClusterSteal<F>::value) {
      // cluster work stealing (VP_FLAG_CLUSTER_STEAL): the cooperative megakernel as
      // clusters of 2 CTAs; if the driver refuses, the plain cooperative launch (the kernel
      // then sees a cluster of 1 and does not steal)
      if (coop && (c.flags & FLAG_STEAL) && grid % 2 == 0) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = blk;
        cfg.dynamicSmemBytes = sm;
        cfg.stream = st;
        cudaLaunchAttribute at[2];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = 2;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        at[1].id = cudaLaunchAttributeCooperative;
        at[1].val.cooperative = 1;
        cfg.attrs = at;
        cfg.numAttrs = 2;
        if (cudaLaunchKernelExC(&cfg, k, args) == cudaSuccess) return cudaSuccess;
        (void)cudaGetLastError();
      }
    }
    if (coop) return cudaLaunchCooperativeKernel(k, dim3(grid), blk, args, sm, st);
    return cudaLaunchKernel(k, dim3(grid), blk, args, sm, st);
  }
  cudaError_t init_run(const void* params, cudaStream_t st) const override {
    return F::init_run(*(const typename F::Params*)params, st);
  }
  cudaError_t finalize(const void* params, cudaStream_t st) const override {
    return F::finalize(*(const typename F::Params*)params, st);
  }
  bool output(const void* params, int idx, void** ptr, size_t* bytes) const override {
    return F::output(*(const typename F::Params*)params, idx, ptr, bytes);
  }
  const char* validate(const void* params) const override { return F::validate(*(const typename F::Params*)params); }
};

// Family accessors (one per family translation unit).
const FamilyOps* family_toy();
const FamilyOps* family_collatz();
const FamilyOps* family_reyes();
const FamilyOps* family_raster();
const FamilyOps* family_pyramid();
const FamilyOps* family_cfd();
const FamilyOps* family_facedet();
const FamilyOps* family_qbench4();
const FamilyOps* family_qbench16();
const FamilyOps* family_qbench272();
const FamilyOps* family_qbench4_cs();
const FamilyOps* family_qbench16_cs();
const FamilyOps* family_ldpc();

}  // namespace vp
