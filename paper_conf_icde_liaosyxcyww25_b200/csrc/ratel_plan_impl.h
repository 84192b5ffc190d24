// ratel_plan_impl.h -- library-internal glue between the host-only planner
// (ratel_plan.cpp) and the runtime's thread-local error message.
#pragma once

namespace ratel {
// Sets ratel_last_error()'s message; returns `code`.
int report_error(int code, const char* msg);
}  // namespace ratel
