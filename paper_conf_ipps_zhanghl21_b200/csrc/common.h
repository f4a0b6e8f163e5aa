// Internal types of libduet (host side).  The public boundary is include/duet.h.
#pragma once

#include <cstdint>
#include <map>
#include <memory>
#include <set>
#include <string>
#include <functional>
#include <vector>

#include "duet.h"

namespace duet {

struct Error {
  duet_status code;
  std::string msg;
};
[[noreturn]] inline void fail(duet_status c, const std::string& m) { throw Error{c, m}; }

enum DType { kF32 = 0, kBF16 = 1, kI32 = 2, kI64 = 3 };
inline int dtype_bytes(int d) { return d == kF32 ? 4 : d == kBF16 ? 2 : d == kI32 ? 4 : 8; }
const char* dtype_name(int d);

struct Node {
  int id = 0;
  std::string name, op;
  std::vector<std::pair<char, std::string>> args;  // ('%'|'@', name) in argument order
  std::map<std::string, std::string> attrs;
  int dtype = kF32;
  std::vector<int64_t> shape;
  std::vector<int> inputs;      // unique producer node ids, ascending
  std::vector<int> arg_nodes;   // producer of each %-argument, in argument order
  std::vector<std::string> params;  // @-arguments in order
  int64_t numel() const {
    int64_t n = 1;
    for (auto s : shape) n *= s;
    return n;
  }
  int64_t nbytes() const { return numel() * dtype_bytes(dtype); }
  int64_t attr_int(const std::string& k, int64_t dflt) const;
  std::string attr_str(const std::string& k, const std::string& dflt) const;
};

struct ParamDecl {
  int dtype = kF32;
  std::vector<int64_t> shape;
  int64_t numel() const {
    int64_t n = 1;
    for (auto s : shape) n *= s;
    return n;
  }
};

struct Binding {
  void* data = nullptr;
  int device = -1;
};

struct Program;  // device-side executable (runtime.cu)

struct Graph {
  std::vector<Node> nodes;
  std::map<std::string, ParamDecl> params;
  std::vector<std::string> param_order;
  std::vector<int> outputs;      // node ids, IR order of the output lines (dedup)
  std::vector<int> input_nodes;  // node ids of op == input, declaration order
  std::map<std::string, int> by_name;
  std::map<std::string, Binding> bound;
  std::vector<int> topo;         // Kahn order, smallest ready id first
  std::shared_ptr<Program> prog; // built lazily by profile / run
  ~Graph();
};

Graph* parse_ir(const char* text, size_t len);

enum PhaseKind { kSeq = 0, kMulti = 1 };

struct Partition {
  const Graph* g = nullptr;
  int granularity = 0;
  std::vector<int> node_to_sg;                 // over IR nodes; -1 = input
  std::vector<std::vector<int>> sg_nodes;      // IR node ids in topological rank order
  std::vector<int> sg_phase;
  std::vector<int> phase_kind;
  std::map<std::pair<int, int>, int64_t> edges;  // (src,dst) -> bytes; -1 = graph in/out
  int n_placeholders = 0;
  int batch_shards = 1;
  std::vector<int> sg_shard;   // row-shard index of each subgraph, -1 = unsharded
  std::vector<int> sg_origin;  // the unsharded subgraph a shard comes from
  int n_sg() const { return (int)sg_nodes.size(); }
  bool sharded() const { return batch_shards > 1; }
};

Partition* make_partition(const Graph* g, int granularity, int batch_shards = 1);

struct Profile {
  const Partition* p = nullptr;
  int n_slots = 0;
  std::vector<int> slot_gpu;
  std::vector<int64_t> t_ns;  // [n_sg * n_slots]
  duet_comm_model comm{};
  int64_t T(int s, int d) const { return t_ns[(size_t)s * n_slots + d]; }
};

struct ExecCache;  // runtime.cu

struct Schedule {
  const Partition* p = nullptr;
  const Profile* pr = nullptr;
  std::vector<int> slot_of;
  std::vector<int> order;
  int64_t makespan = 0;
  int fell_back = 0;
  int64_t measured_ns = -1;         // measured mode: device latency of slot_of (else -1)
  int trace = 0;                    // 1: duet_run records per-subgraph start / end events
  std::shared_ptr<ExecCache> exec;  // captured CUDA graphs (runtime.cu)
  ~Schedule();
};

// latency of a complete assignment (slot per subgraph), int64 ns
using Latency = std::function<int64_t(const std::vector<int>&)>;

Schedule* make_schedule(const Partition* p, const Profile* pr, const duet_sched_opts* o);
// Same algorithm; Step 3's and the fallback's `measure latency` = `measured` when non-null.
Schedule* make_schedule_with(const Partition* p, const Profile* pr, const duet_sched_opts* o,
                             const Latency* measured);
// Measured mode: times each candidate assignment on the device.
Schedule* schedule_measured(const Partition* p, const Profile* pr, const duet_sched_opts* o,
                            const duet_slot* slots, int n_slots, duet_measure_opts* mo);

// ---- runtime (runtime.cu) ----
Profile* profile_on_device(const Partition* p, const duet_slot* slots, int n_slots,
                           const duet_profile_opts* o);
void run_schedule(Schedule* s, const duet_slot* slots, int n_slots, const duet_tensor* in, int n_in,
                  duet_tensor* out, int n_out);
int64_t schedule_launch_count(const Schedule* s);
// per-subgraph [start, end) of the last traced duet_run, ns after its fork (waits for that run)
void schedule_trace_export(const Schedule* s, int64_t* start_ns, int64_t* end_ns, int n);
void node_run(Graph* g, const std::string& node, const duet_tensor* args, int n_args, duet_tensor* out,
              void* stream);
void destroy_program(Program* p);
void destroy_exec(ExecCache* e);

}  // namespace duet
