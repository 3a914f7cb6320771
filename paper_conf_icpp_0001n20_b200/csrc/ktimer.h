// ktimer.h -- CUDA-event timing of one kernel across the launches of a run
// (profile mode: eager launches, an event pair around each launch).
#pragma once
#include <cuda_runtime.h>

#include <vector>

namespace gx {
struct KTimer {
  bool on = false;
  cudaStream_t s = nullptr;
  std::vector<cudaEvent_t> ev;
  explicit KTimer(bool enable, cudaStream_t st) : on(enable), s(st) {}
  void begin() {
    if (!on) return;
    cudaEvent_t e;
    cudaEventCreate(&e);
    cudaEventRecord(e, s);
    ev.push_back(e);
  }
  void end() { begin(); }
  int launches() const { return (int)ev.size() / 2; }
  double total_ms() {
    double t = 0;
    if (!on) return 0;
    cudaStreamSynchronize(s);
    for (size_t i = 0; i + 1 < ev.size(); i += 2) {
      float ms = 0;
      cudaEventElapsedTime(&ms, ev[i], ev[i + 1]);
      t += ms;
    }
    return t;
  }
  ~KTimer() {
    for (auto e : ev) cudaEventDestroy(e);
  }
};
}  // namespace gx
