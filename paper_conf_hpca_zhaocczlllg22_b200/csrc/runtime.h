// runtime.h — internal host-side declarations shared by the C ABI translation units.
#pragma once
#include <string>

#include "tacker.h"

namespace tkrt {

void set_error(const char *fmt, ...);
tacker_status cuda_fail(const char *what, int err);
int sm_count();

// model store (predictor.cpp)
bool model_predict(const std::string &key, double x, double *y);
bool pair_predict(const std::string &key, double x_tc, double x_cd, double *y);
bool pair_opportune(const std::string &key, double *r);

// register-rich fused instantiations (fused_rich.cu): fused_kernel<BN, kind, 8> or nullptr
void *pick_fused_rich(int BN, int be_kind);

// LC-only kernels per (BN, LC mode, epilogue 1 = TMA store / 2 = register) (fused_lc.cu) or nullptr
void *pick_lc_only_kernel(int BN, int mode, int epi);

// default-class fused kernels per (BN, BE kind, LC mode) for the bench's kinds (fused_mode.cu) or nullptr
void *pick_fused_mode_kernel(int BN, int be_kind, int mode);

// kind names
const char *be_kind_name(int kind);

}  // namespace tkrt
