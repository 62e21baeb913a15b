// nvml_dyn.h -- NVML loaded at run time (dlopen), so libsph loads on hosts
// without a driver (the CPU build box) and energy accounting degrades to
// "unavailable" instead of failing.  Used for the paper's per-function energy
// (energy from the start of each function to its completion) and clock
// control (NVML clock set before each function).
#pragma once
#include <stdint.h>

namespace sph {

struct Nvml {
  bool ok = false;              // library loaded, initialised, device found
  bool energy_ok = false;       // total-energy counter readable
  void* lib = nullptr;
  void* dev = nullptr;          // nvmlDevice_t
  int last_rc = 0;
  char err[160] = {0};

  bool init(int cuda_device);   // maps the CUDA device to NVML by PCI bus id
  void shutdown();
  bool energy_mj(unsigned long long* mj);
  bool sm_clock_mhz(unsigned* mhz);
  bool power_mw(unsigned* mw);          // nvmlDeviceGetPowerUsage (~1 s average)
  bool power_instant_mw(unsigned* mw);  // field NVML_FI_DEV_POWER_INSTANT (fast read; B200 updates it ~every 100 ms)
  int supported_sm_clocks(unsigned* out, unsigned cap);  // returns count (<= cap)
  int lock_sm_clock(unsigned mhz);  // 0 ok, else NVML return code
  int reset_sm_clock();
  const char* error_string(int rc);
};

}  // namespace sph
