// errors.h — thread-local last-error message behind arlo_last_error().
#pragma once

namespace arlo {
// Record a printf-style message for the calling thread and return `code`.
int set_error(int code, const char* fmt, ...);
void clear_error();
}  // namespace arlo
