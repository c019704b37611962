// common.h -- internal helpers shared by the C-ABI translation units of libxk.so.
#pragma once
#include <string>

#include "plan/plan.h"
#include "xk.h"

namespace xk {
void set_error(const std::string &msg);
bool make_topology(const xk_topo_t *t, Topology *out, std::string &err);
bool make_flags(const xk_flags_t *f, int G, Flags *out, std::string &err);
void default_grid(int G, int *P, int *Q);
}  // namespace xk
