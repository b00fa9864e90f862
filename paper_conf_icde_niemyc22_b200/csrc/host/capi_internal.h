// Definitions of the opaque C-ABI handles.
#pragma once
#include "core.h"

struct ts_graph_s {
  ts::Graph g;
};
struct ts_profile_s {
  ts::Profile pr;
};
struct ts_plan_s {
  const ts::Graph* graph = nullptr;
  ts::PlanState st;
  uint64_t budget = 0;
};
