// Opaque C-ABI handles (include/adainf.h) wrapping the runtime objects; shared by the API translation units.
#pragma once
#include "model.h"

struct adainf_model {
  adainf::Model m;
};
struct adainf_app {
  adainf::App a;
};
