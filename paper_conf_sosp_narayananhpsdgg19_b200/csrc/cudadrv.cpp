// cudadrv.cpp -- driver-API entry points resolved at run time through the runtime's
// cudaGetDriverEntryPoint, so libpipedream.so has no link-time dependency on libcuda.so
// (it must load -- and fail loudly on use -- on a machine without a GPU driver).
#include <mutex>

#include "pd_internal.h"

namespace pd {

const Driver *driver() {
    static Driver d;
    static bool ok = false;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q1{}, q2{};
        void *f1 = nullptr, *f2 = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &f1, cudaEnableDefault, &q1) != cudaSuccess) f1 = nullptr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f2, cudaEnableDefault, &q2) != cudaSuccess) f2 = nullptr;
        d.streamWaitValue32 = reinterpret_cast<decltype(d.streamWaitValue32)>(f1);
        d.tensorMapEncodeTiled = reinterpret_cast<decltype(d.tensorMapEncodeTiled)>(f2);
        ok = f1 && f2;
        cudaGetLastError();
    });
    return ok ? &d : nullptr;
}

}  // namespace pd
