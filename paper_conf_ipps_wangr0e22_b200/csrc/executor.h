// executor.h — replays a Plan on the GPUs (see executor.cu).
#pragma once

#include <memory>

#include "core.h"

namespace micco {

micco_status nccl_unique_id(uint8_t out[128]);

class Executor {
 public:
  explicit Executor(Context &c);
  ~Executor();
  void execute(int n_gpus, const int32_t *reuse_bound);
  void fetch_graph_values();
  void release_cache();
  struct Impl;

 private:
  std::unique_ptr<Impl> p_;
};

}  // namespace micco
