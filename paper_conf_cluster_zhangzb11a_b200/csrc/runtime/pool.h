// A small persistent host thread pool for the runtime's embarrassingly parallel host steps
// (candidate generation, trie planning, thresholding).  parallel_for(n, f) runs f(0..n-1) on the
// pool's workers plus the calling thread and returns when all are done.  Calls are serialised
// (one parallel region at a time); nested calls run serially.
#pragma once
#include <cstddef>
#include <functional>

namespace gpa {
size_t pool_threads();
void parallel_for(size_t n, const std::function<void(size_t)>& f);
// host tracing (GPA_TRACE=1) and wall clock; declared for the runtime in internal.h as well
bool trace_enabled();
double wall_ms();
}  // namespace gpa
