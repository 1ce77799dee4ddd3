// status.cu — error strings, thread-local error detail, device capability check.
#include <stdarg.h>
#include <string.h>

#include "common.cuh"

namespace otif {

static thread_local char g_err[512] = "";

void set_error(const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

otif_status check_device(int *num_sms) {
    static int cached_dev = -1, cached_sms = 0, cached_ok = 0;
    int dev = 0;
    OTIF_CUDA(cudaGetDevice(&dev));
    if (dev != cached_dev) {
        cudaDeviceProp prop;
        OTIF_CUDA(cudaGetDeviceProperties(&prop, dev));
        cached_ok = (prop.major == 10 && prop.minor == 0);
        cached_sms = prop.multiProcessorCount;
        cached_dev = dev;
        if (!cached_ok) set_error("device %d is sm_%d%d; libotif is built for sm_100a only", dev, prop.major, prop.minor);
    }
    if (!cached_ok) return OTIF_EUNSUPPORTED;
    if (num_sms) *num_sms = cached_sms;
    return OTIF_OK;
}

}  // namespace otif

extern "C" const char *otif_status_str(otif_status s) {
    switch (s) {
        case OTIF_OK: return "OTIF_OK";
        case OTIF_EINVAL: return "OTIF_EINVAL";
        case OTIF_ENOMEM: return "OTIF_ENOMEM";
        case OTIF_ECUDA: return "OTIF_ECUDA";
        case OTIF_EUNSUPPORTED: return "OTIF_EUNSUPPORTED";
    }
    return "OTIF_UNKNOWN";
}

extern "C" const char *otif_last_error(void) { return otif::g_err; }

extern "C" const char *otif_version(void) { return "otif-b200 0.1 sm_100a"; }
