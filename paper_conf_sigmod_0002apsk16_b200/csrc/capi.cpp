// Error plumbing and version for the C ABI (include/gts.h).
#include <cstdarg>
#include <cstdio>

#include "gts_internal.h"

namespace gts {

static thread_local char t_err[1024] = "";

int fail(int code, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    std::vsnprintf(t_err, sizeof(t_err), fmt, ap);
    va_end(ap);
    return code;
}

void clear_error() { t_err[0] = '\0'; }

}  // namespace gts

extern "C" const char* gts_last_error(void) { return gts::t_err; }
extern "C" int gts_version(void) { return GTS_VERSION; }
