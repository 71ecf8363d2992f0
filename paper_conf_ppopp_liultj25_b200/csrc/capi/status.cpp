#include "status.h"

namespace mario { const char* last_error_cstr(); }

namespace mario {
namespace {
thread_local std::string g_last_error;
}
const char* last_error_cstr() { return g_last_error.c_str(); }

mario_status set_error(mario_status code, const std::string& msg) {
  g_last_error = msg;
  return code;
}

}  // namespace mario

extern "C" const char* mario_last_error(void) { return mario::last_error_cstr(); }
