// status.h — thread-local error message plumbing for the C ABI (include/moment.h conventions).
#pragma once
#include <cstdarg>
#include <cstdio>
#include <string>

#include "moment.h"

namespace moment {

void set_error(const char* fmt, ...);
const char* last_error();

// fail(code, fmt, ...) records a message and returns the code.
inline moment_status fail(moment_status code, const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    set_error("%s", buf);
    return code;
}

}  // namespace moment

#define MOMENT_TRY(expr)                        \
    do {                                        \
        moment_status _st = (expr);             \
        if (_st != MOMENT_OK) return _st;       \
    } while (0)
