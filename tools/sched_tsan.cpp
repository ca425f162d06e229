// ThreadSanitizer harness for the master's task-allocation core (csrc/sched.cpp; SURVEY §5:
// "TSan on the scheduler's ... tests").  Built by tests/test_sched_tsan.py with
//   g++ -std=c++17 -O1 -g -fsanitize=thread -pthread tools/sched_tsan.cpp csrc/sched.cpp
// Worker threads drive one sw_sched the way libsw's workers do: long-poll requests, start,
// progress reports, complete (first result wins), abandon a replica whose task finished
// elsewhere (WA), one worker slowed 6x, one worker failing mid-run.  Checks at the end:
// every task finished and committed exactly once; prints "sched tsan ok".
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <thread>
#include <vector>
#include "../include/sw.h"
#include "../include/sw_sched.h"

static double now_s() {
  using namespace std::chrono;
  static const auto t0 = steady_clock::now();
  return duration<double>(steady_clock::now() - t0).count();
}

int main(int argc, char **argv) {
  const int n_workers = argc > 1 ? atoi(argv[1]) : 6, n_units = argc > 2 ? atoi(argv[2]) : 120;
  for (int policy : {SW_POLICY_SS, SW_POLICY_PSS}) {
    for (int wa : {0, 1}) {
      std::vector<int64_t> cells(n_units);
      for (int u = 0; u < n_units; u++) cells[u] = 1000000 + (int64_t)(u * 7919 % 13) * 200000;
      sw_sched *s = sw_sched_create(n_workers, n_units, cells.data(), policy, wa, 4);
      if (!s) { printf("create failed\n"); return 1; }
      std::vector<std::atomic<int>> commits(n_units);
      for (auto &c : commits) c = 0;
      auto worker = [&](int w) {
        const int slow = (w == n_workers - 1) ? 6 : 1;          // a slower PE
        const bool fails = w == n_workers - 2;                 // gone after a few tasks
        int done = 0;
        int32_t buf[64];
        while (true) {
          const int32_t r = sw_sched_request_wait(s, w, now_s(), buf, 64, 0.005);
          if (r < 0) break;
          for (int32_t i = 0; i < r; i++) {
            const int u = buf[i];
            if (!sw_sched_start(s, w, u, now_s())) continue;
            const double t0 = now_s();
            bool cancelled = false;
            for (int step = 0; step < 4 * slow; step++) {   // "compute", polling for cancellation
              std::this_thread::sleep_for(std::chrono::microseconds(50 + (u % 5) * 20));
              if (sw_sched_is_finished(s, u)) { cancelled = true; break; }
            }
            if (cancelled) {
              sw_sched_abandon(s, w, u, now_s());
            } else {
              if (sw_sched_complete(s, w, u, now_s())) commits[u]++;
              sw_sched_report(s, w, now_s(), (double)cells[u], now_s() - t0);
            }
            if (fails && ++done == 3) {
              sw_sched_fail_worker(s, w, now_s());
              return;
            }
          }
        }
      };
      std::vector<std::thread> ts;
      for (int w = 0; w < n_workers; w++) ts.emplace_back(worker, w);
      for (auto &t : ts) t.join();
      for (int u = 0; u < n_units; u++) {
        if (!sw_sched_is_finished(s, u) || commits[u] != 1 || sw_sched_committed_by(s, u) < 0) {
          printf("unit %d: finished %d commits %d (policy %d, wa %d)\n", u, sw_sched_is_finished(s, u),
                 (int)commits[u], policy, wa);
          return 1;
        }
      }
      printf("policy %d wa %d: %lld requests, %lld WA grants\n", policy, wa, (long long)sw_sched_counter(s, 0),
             (long long)sw_sched_counter(s, 1));
      sw_sched_destroy(s);
    }
  }
  printf("sched tsan ok\n");
  return 0;
}
