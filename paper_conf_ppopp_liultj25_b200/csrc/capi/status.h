// Thread-local error string + exception guard: no C++ exception crosses the C-ABI.
#pragma once
#include <exception>
#include <memory>
#include <string>

#include "../../../include/mario.h"

namespace mario {

mario_status set_error(mario_status code, const std::string& msg);

template <class F>
mario_status guard(F&& f) {
  try {
    return f();
  } catch (const std::bad_alloc&) {
    return set_error(MARIO_EINVAL, "host out of memory");
  } catch (const std::exception& e) {
    return set_error(MARIO_EINVAL, e.what());
  } catch (...) {
    return set_error(MARIO_EINVAL, "unknown exception");
  }
}

}  // namespace mario
