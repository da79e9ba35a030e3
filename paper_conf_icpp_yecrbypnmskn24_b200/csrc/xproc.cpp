// xproc.cpp -- cross-process channel (one process per GPU).  Filled in below
// the in-process path; until then registration reports VIPER_E_UNSUPPORTED.
#include "runtime.h"

using namespace vp;

extern "C" viper_status viper_xproc_register(viper_model *m, const viper_tensor *, const viper_bootstrap *) {
    (void)m;
    return set_error(VIPER_E_UNSUPPORTED, "cross-process channel not built yet");
}

extern "C" viper_status viper_xproc_publish(viper_model *, uint64_t, cudaStream_t) {
    return set_error(VIPER_E_UNSUPPORTED, "cross-process channel not built yet");
}
