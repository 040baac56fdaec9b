// NVSwitch multicast data plane ("push" = 2, NEXT-3, PAPER.md:216 / :471): the
// replicas of every pushed tile live in ONE multicast object bound on all devices
// of the call, at the same offset on every device; the producing kernel's
// epilogue writes each finished element once with multimem.st and the switch
// delivers it to every device.  One slab of (pushed tiles) x nb^2 doubles per
// device (17.4 GB at n = 65536: B200's 180 GB holds it); devices that do not read
// a tile simply receive an unused copy -- NVLink ingress stays far below the link
// rate (<= 10.6 GB of panel traffic into a GPU per factorisation).
// Eligibility: >= 2 slots on distinct devices, single-process mode, and every
// device reports CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED; otherwise (and on any
// driver error) the call keeps the per-replica peer stores of "push" = 1.
#include <cstring>

#include "runtime_internal.hpp"

namespace stfrt {

namespace {
struct Drv {
  CUresult (*attr)(int*, CUdevice_attribute, CUdevice) = nullptr;
  CUresult (*gran)(size_t*, const CUmulticastObjectProp*, CUmulticastGranularity_flags) = nullptr;
  CUresult (*create)(CUmemGenericAllocationHandle*, const CUmulticastObjectProp*) = nullptr;
  CUresult (*add)(CUmemGenericAllocationHandle, CUdevice) = nullptr;
  CUresult (*bind)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                   unsigned long long) = nullptr;
  CUresult (*unbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t) = nullptr;
  CUresult (*memcreate)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long) =
      nullptr;
  CUresult (*reserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long) = nullptr;
  CUresult (*map)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long) = nullptr;
  CUresult (*access)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t) = nullptr;
  CUresult (*unmap)(CUdeviceptr, size_t) = nullptr;
  CUresult (*release)(CUmemGenericAllocationHandle) = nullptr;
  CUresult (*vfree)(CUdeviceptr, size_t) = nullptr;
  bool ok = false;
};

template <class F>
bool sym(const char* name, F& f) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess)
    return false;
  f = reinterpret_cast<F>(p);
  return true;
}

const Drv& drv() {
  static Drv d = [] {
    Drv x;
    x.ok = sym("cuDeviceGetAttribute", x.attr) && sym("cuMulticastGetGranularity", x.gran) &&
           sym("cuMulticastCreate", x.create) && sym("cuMulticastAddDevice", x.add) &&
           sym("cuMulticastBindMem", x.bind) && sym("cuMulticastUnbind", x.unbind) && sym("cuMemCreate", x.memcreate) &&
           sym("cuMemAddressReserve", x.reserve) && sym("cuMemMap", x.map) && sym("cuMemSetAccess", x.access) &&
           sym("cuMemUnmap", x.unmap) && sym("cuMemRelease", x.release) && sym("cuMemAddressFree", x.vfree);
    return x;
  }();
  return d;
}
}  // namespace

McSlab::~McSlab() {
  const Drv& d = drv();
  if (!d.ok) return;
  if (mcva) {
    d.unmap(mcva, size);
    d.vfree(mcva, size);
  }
  for (size_t k = 0; k < devs.size(); ++k) {
    if (k < uc.size() && uc[k]) {
      d.unmap(uc[k], size);
      d.vfree(uc[k], size);
    }
    if (bound.size() > k && bound[k]) d.unbind(mc, (CUdevice)devs[k], 0, size);
    if (k < phys.size() && phys[k]) d.release(phys[k]);
  }
  if (mc) d.release(mc);
}

// Every device of `devs` supports multicast objects (and the driver exports the API).
bool mc_supported(const std::vector<int>& devs, std::string* why) {
  const Drv& d = drv();
  if (!d.ok) {
    *why = "driver lacks the multicast API";
    return false;
  }
  if (devs.size() < 2) {
    *why = "multicast needs >= 2 distinct devices";
    return false;
  }
  for (int dev : devs) {
    int v = 0;
    if (d.attr(&v, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, (CUdevice)dev) != CUDA_SUCCESS || !v) {
      *why = "device " + std::to_string(dev) + " does not support multicast objects";
      return false;
    }
  }
  return true;
}

// One multicast object of `bytes` (rounded up to the granularity) bound on every
// device of `devs`; uc[k] is device k's own mapping of its copy, mcva the
// multicast mapping (accessible from every device).
int mc_create(McSlab& S, const std::vector<int>& devs, size_t bytes, std::string* why) {
  const Drv& d = drv();
  S.devs = devs;
  CUmulticastObjectProp prop;
  memset(&prop, 0, sizeof prop);
  prop.numDevices = (unsigned)devs.size();
  prop.handleTypes = CU_MEM_HANDLE_TYPE_NONE;
  prop.size = bytes;
  size_t g = 0;
  if (d.gran(&g, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS || !g) {
    *why = "cuMulticastGetGranularity failed";
    return -1;
  }
  S.size = prop.size = (bytes + g - 1) / g * g;
  if (d.create(&S.mc, &prop) != CUDA_SUCCESS) {
    *why = "cuMulticastCreate failed";
    return -1;
  }
  for (int dev : devs)
    if (d.add(S.mc, (CUdevice)dev) != CUDA_SUCCESS) {
      *why = "cuMulticastAddDevice failed";
      return -1;
    }
  S.phys.assign(devs.size(), 0);
  S.uc.assign(devs.size(), 0);
  S.bound.assign(devs.size(), 0);
  for (size_t k = 0; k < devs.size(); ++k) {
    CUmemAllocationProp ap;
    memset(&ap, 0, sizeof ap);
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = devs[k];
    if (d.memcreate(&S.phys[k], S.size, &ap, 0) != CUDA_SUCCESS) {
      *why = "cuMemCreate failed (device memory)";
      return -103;
    }
    if (d.bind(S.mc, 0, S.phys[k], 0, S.size, 0) != CUDA_SUCCESS) {
      *why = "cuMulticastBindMem failed";
      return -1;
    }
    S.bound[k] = 1;
    CUmemAccessDesc ad;
    ad.location = ap.location;
    ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    if (d.reserve(&S.uc[k], S.size, g, 0, 0) != CUDA_SUCCESS || d.map(S.uc[k], S.size, 0, S.phys[k], 0) != CUDA_SUCCESS ||
        d.access(S.uc[k], S.size, &ad, 1) != CUDA_SUCCESS) {
      *why = "mapping a device's multicast copy failed";
      return -1;
    }
  }
  std::vector<CUmemAccessDesc> acc(devs.size());
  for (size_t k = 0; k < devs.size(); ++k) {
    acc[k].location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    acc[k].location.id = devs[k];
    acc[k].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  }
  if (d.reserve(&S.mcva, S.size, g, 0, 0) != CUDA_SUCCESS || d.map(S.mcva, S.size, 0, S.mc, 0) != CUDA_SUCCESS ||
      d.access(S.mcva, S.size, acc.data(), acc.size()) != CUDA_SUCCESS) {
    *why = "mapping the multicast address range failed";
    return -1;
  }
  return 0;
}

}  // namespace stfrt
