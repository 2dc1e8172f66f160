// special.cpp -- modexp (row a8) and sin_taylor (row a9) specialisations.
#include <cuda_runtime.h>

#include <mutex>
#include <string>

#include "../../include/up.h"
#include "codegen.h"
#include "hbig.h"
#include "up_kparams.h"

using namespace uph;

up_status up_internal_fail(up_status st, const std::string &msg);

extern "C" {

up_status up_modexp(up_ctx *, const up_column *, const char *, const char *, up_column *, void *) {
    return up_internal_fail(UP_E_UNSUPPORTED, "up_modexp: not built yet");
}
up_status up_modexp_sum_type(up_ctx *, const char *, int64_t, int32_t *, int32_t *) {
    return up_internal_fail(UP_E_UNSUPPORTED, "up_modexp_sum_type: not built yet");
}
up_status up_modexp_sum(up_ctx *, const up_column *, const char *, const char *, int64_t, uint32_t *, void *) {
    return up_internal_fail(UP_E_UNSUPPORTED, "up_modexp_sum: not built yet");
}
up_status up_sin_taylor(up_ctx *, const up_column *, int32_t, up_column *, void *) {
    return up_internal_fail(UP_E_UNSUPPORTED, "up_sin_taylor: not built yet");
}
up_status up_sin_taylor_sum(up_ctx *, const up_column *, int32_t, int64_t, uint32_t *, void *) {
    return up_internal_fail(UP_E_UNSUPPORTED, "up_sin_taylor_sum: not built yet");
}

}  // extern "C"
