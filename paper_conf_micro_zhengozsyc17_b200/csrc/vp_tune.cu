// vp_tune.cu — placeholder, replaced by the auto-tuner below in this file's next revision.
#include "../../include/vp.h"
extern "C" {
vp_status vp_autotune(void*, const vp_autotune_opts*, vp_config*, vp_tune_report*) { return VP_ERR_UNSUPPORTED; }
vp_status vp_config_to_string(const vp_config*, char*, size_t) { return VP_ERR_UNSUPPORTED; }
vp_status vp_config_from_string(const char*, vp_config*) { return VP_ERR_UNSUPPORTED; }
}
