// nvml_dyn.cpp -- see nvml_dyn.h.  Prototypes follow /usr/local/cuda/include/nvml.h
// (nvmlDeviceGetTotalEnergyConsumption nvml.h:6024, nvmlDeviceGetClockInfo :5042,
// nvmlDeviceGetPowerUsage :6006, nvmlDeviceGetSupportedGraphicsClocks :5212,
// nvmlDeviceSetGpuLockedClocks :8169, nvmlDeviceResetGpuLockedClocks :8191).
#include "nvml_dyn.h"

#include <cuda_runtime.h>
#include <dlfcn.h>
#include <stdio.h>
#include <string.h>

namespace sph {

namespace {
typedef int (*fn_init)(void);
typedef int (*fn_shutdown)(void);
typedef int (*fn_by_pci)(const char*, void**);
typedef int (*fn_energy)(void*, unsigned long long*);
typedef int (*fn_clock)(void*, int, unsigned*);
typedef int (*fn_power)(void*, unsigned*);
typedef int (*fn_sup_mem)(void*, unsigned*, unsigned*);
typedef int (*fn_sup_gr)(void*, unsigned, unsigned*, unsigned*);
typedef int (*fn_lock)(void*, unsigned, unsigned);
typedef int (*fn_reset)(void*);
typedef const char* (*fn_errstr)(int);
// nvmlFieldValue_t (nvml.h:2677): fieldId, scopeId, timestamp, latencyUsec,
// valueType, nvmlReturn, value (8-byte union)
struct FieldValue {
  unsigned fieldId, scopeId;
  long long timestamp, latencyUsec;
  int valueType, nvmlReturn;
  unsigned long long value;
};
typedef int (*fn_fields)(void*, int, FieldValue*);
constexpr unsigned kFiPowerInstant = 186;  // NVML_FI_DEV_POWER_INSTANT (nvml.h:2496)

struct Syms {
  fn_init init;
  fn_shutdown shutdown;
  fn_by_pci by_pci;
  fn_energy energy;
  fn_clock clock;
  fn_power power;
  fn_sup_mem sup_mem;
  fn_sup_gr sup_gr;
  fn_lock lock;
  fn_reset reset;
  fn_errstr errstr;
  fn_fields fields;
};
Syms g_syms;
constexpr int kNvmlClockSM = 1;  // NVML_CLOCK_SM
}  // namespace

bool Nvml::init(int cuda_device) {
  lib = dlopen("libnvidia-ml.so.1", RTLD_NOW | RTLD_LOCAL);
  if (!lib) {
    snprintf(err, sizeof(err), "libnvidia-ml.so.1 not loadable");
    return false;
  }
  g_syms.init = (fn_init)dlsym(lib, "nvmlInit_v2");
  g_syms.shutdown = (fn_shutdown)dlsym(lib, "nvmlShutdown");
  g_syms.by_pci = (fn_by_pci)dlsym(lib, "nvmlDeviceGetHandleByPciBusId_v2");
  g_syms.energy = (fn_energy)dlsym(lib, "nvmlDeviceGetTotalEnergyConsumption");
  g_syms.clock = (fn_clock)dlsym(lib, "nvmlDeviceGetClockInfo");
  g_syms.power = (fn_power)dlsym(lib, "nvmlDeviceGetPowerUsage");
  g_syms.sup_mem = (fn_sup_mem)dlsym(lib, "nvmlDeviceGetSupportedMemoryClocks");
  g_syms.sup_gr = (fn_sup_gr)dlsym(lib, "nvmlDeviceGetSupportedGraphicsClocks");
  g_syms.lock = (fn_lock)dlsym(lib, "nvmlDeviceSetGpuLockedClocks");
  g_syms.reset = (fn_reset)dlsym(lib, "nvmlDeviceResetGpuLockedClocks");
  g_syms.errstr = (fn_errstr)dlsym(lib, "nvmlErrorString");
  g_syms.fields = (fn_fields)dlsym(lib, "nvmlDeviceGetFieldValues");
  if (!g_syms.init || !g_syms.by_pci) {
    snprintf(err, sizeof(err), "NVML symbols missing");
    return false;
  }
  last_rc = g_syms.init();
  if (last_rc != 0) {
    snprintf(err, sizeof(err), "nvmlInit failed: %d", last_rc);
    return false;
  }
  char bus[64] = {0};
  if (cudaDeviceGetPCIBusId(bus, sizeof(bus), cuda_device) != cudaSuccess) {
    cudaGetLastError();
    snprintf(err, sizeof(err), "cudaDeviceGetPCIBusId failed");
    return false;
  }
  last_rc = g_syms.by_pci(bus, &dev);
  if (last_rc != 0) {
    snprintf(err, sizeof(err), "nvmlDeviceGetHandleByPciBusId(%s): %d", bus, last_rc);
    return false;
  }
  ok = true;
  unsigned long long e;
  energy_ok = g_syms.energy && g_syms.energy(dev, &e) == 0;
  return true;
}

void Nvml::shutdown() {
  if (ok && g_syms.shutdown) g_syms.shutdown();
  ok = false;
  // the library stays loaded (dlclose of NVML while other users hold it is unsafe)
}

bool Nvml::energy_mj(unsigned long long* mj) {
  if (!energy_ok) return false;
  return (last_rc = g_syms.energy(dev, mj)) == 0;
}

bool Nvml::sm_clock_mhz(unsigned* mhz) {
  if (!ok || !g_syms.clock) return false;
  return (last_rc = g_syms.clock(dev, kNvmlClockSM, mhz)) == 0;
}

bool Nvml::power_mw(unsigned* mw) {
  if (!ok || !g_syms.power) return false;
  return (last_rc = g_syms.power(dev, mw)) == 0;
}

bool Nvml::power_instant_mw(unsigned* mw) {
  if (!ok || !g_syms.fields) return false;
  FieldValue v{};
  v.fieldId = kFiPowerInstant;
  if ((last_rc = g_syms.fields(dev, 1, &v)) != 0) return false;
  if (v.nvmlReturn != 0) {
    last_rc = v.nvmlReturn;
    return false;
  }
  *mw = (unsigned)v.value;  // unsigned int member of the union (little endian)
  return true;
}

int Nvml::supported_sm_clocks(unsigned* out, unsigned cap) {
  if (!ok || !g_syms.sup_mem || !g_syms.sup_gr) return 0;
  unsigned nmem = 8, mem[8];
  if (g_syms.sup_mem(dev, &nmem, mem) != 0 || nmem == 0) return 0;
  unsigned n = cap;
  if ((last_rc = g_syms.sup_gr(dev, mem[0], &n, out)) != 0) return 0;
  return (int)n;
}

int Nvml::lock_sm_clock(unsigned mhz) {
  if (!ok || !g_syms.lock) return -1;
  return last_rc = g_syms.lock(dev, mhz, mhz);
}

int Nvml::reset_sm_clock() {
  if (!ok || !g_syms.reset) return -1;
  return last_rc = g_syms.reset(dev);
}

const char* Nvml::error_string(int rc) {
  if (g_syms.errstr) return g_syms.errstr(rc);
  return "NVML unavailable";
}

}  // namespace sph
