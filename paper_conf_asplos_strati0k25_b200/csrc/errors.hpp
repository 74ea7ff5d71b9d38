// errors.hpp — thread-local error detail for pcc_last_error / pcc_last_errno.
#pragma once
#include <cstdio>
#include <cstring>
#include <string>

namespace pcc {

struct ErrState {
    std::string msg;
    int err_no = 0;
};
inline ErrState &err_state() {
    static thread_local ErrState s;
    return s;
}
// returns -code so callers can `return set_error(...)`
inline int set_error(int code, const char *what) {
    err_state().msg = what ? what : "";
    return -code;
}
inline int set_errno_error(const char *what, int e) {
    char b[256];
    std::snprintf(b, sizeof b, "%s: %s", what, std::strerror(e));
    err_state().msg = b;
    err_state().err_no = e;
    return -5;  // -PCC_EIO
}

}  // namespace pcc
