// net.h — multi-process control plane: the paper's master/slave messages (P16 §IV:
// "the master process starts the execution and waits for the slaves to register";
// "When the slaves finish the execution of the assigned tasks, they communicate with the
// master, asking for more tasks") carried over TCP between the processes of one node
// (torchrun, one process per GPU).  The master runs as threads inside rank 0 and owns
// the sw_sched task table; every rank (rank 0 included) is a slave/client.
#pragma once
#include <atomic>
#include <cstdint>
#include <mutex>
#include <string>
#include <thread>
#include <vector>
#include "../../include/sw_sched.h"

namespace sw {

class MasterServer {
 public:
  ~MasterServer();
  // bind 0.0.0.0:port, accept `world` slaves; throws sw::Error-like std::runtime_error
  void start(int port, int world, int32_t n_units, const int64_t *unit_cells, int32_t policy,
             int32_t wa, int32_t omega, uint64_t plan_hash);
  void stop();  // waits for every slave's DONE (or lost connection), then closes
  const std::string &final_log() const { return final_log_; }   // grant log, kept by stop()
 private:
  void serve(int fd);
  int listen_fd_ = -1;
  int world_ = 0;
  sw_sched *sched_ = nullptr;
  std::thread accept_thread_;
  std::vector<std::thread> conns_;
  std::mutex mu_;
  std::atomic<int> done_{0};
  std::atomic<int> registered_{0};
  std::atomic<bool> stopping_{false};
  uint64_t plan_hash_ = 0;
  std::string final_log_ = "[]";
};

class SchedClient {
 public:
  ~SchedClient();
  void connect(const char *host, int port, int rank, double timeout_s, uint64_t plan_hash);
  int32_t request(double t, int32_t *out, int32_t cap);
  int32_t request_wait(double t, int32_t *out, int32_t cap, double timeout_s);   // long poll
  void report(double t, double cells, double sec);
  int32_t complete(int32_t unit, double t);
  void abandon(int32_t unit, double t);
  int32_t start(int32_t unit, double t);   // 1 = run it, 0 = finished or moved away
  int32_t is_finished(int32_t unit);   // cached bitmap, refreshed at most every 0.5 ms
  void done();
  int32_t wa_grants() const { return wa_; }
  int32_t requests() const { return req_; }
  int32_t grant_msgs() const { return grants_; }
  int64_t counter(int32_t which);   // live master counter (kCounters)
 private:
  int32_t call(int32_t op, int32_t unit, int32_t cap, double t, double cells, double sec,
               std::vector<int32_t> *extra, uint64_t hash = 0);
  int fd_ = -1;
  int rank_ = 0;
  std::vector<int32_t> finished_;
  double last_refresh_ = -1;
  int32_t wa_ = 0, req_ = 0, grants_ = 0;
};

}  // namespace sw
