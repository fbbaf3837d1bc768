// Internal interface between ooo_api.cpp and the host modules built on the
// public ABI (pipeline.cpp).  Not part of include/ooo.h.
#pragma once
#include <cuda_runtime.h>

#include "../../include/ooo.h"

namespace ooo {
ooo_status set_error(ooo_status st, const char *msg);          // sets ooo_last_error, returns st
ooo_graph *wrap_graph(cudaGraph_t g, cudaGraphExec_t e);       // ooo_graph_launch / ooo_graph_destroy work on it
}  // namespace ooo
