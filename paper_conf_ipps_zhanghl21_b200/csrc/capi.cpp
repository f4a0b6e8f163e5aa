// C ABI glue (include/duet.h): argument checking, error capture, handle lifetimes.
#include <cstring>

#include "common.h"

using namespace duet;

struct duet_graph_t {
  std::unique_ptr<Graph> g;
};
struct duet_partition_t {
  std::unique_ptr<Partition> p;
};
struct duet_profile_t {
  std::unique_ptr<Profile> pr;
};
struct duet_schedule_t {
  std::unique_ptr<Schedule> s;
};

namespace {
thread_local std::string g_err;

template <class F>
duet_status guard(F&& f) {
  try {
    g_err.clear();
    f();
    return DUET_OK;
  } catch (const Error& e) {
    g_err = e.msg;
    return e.code;
  } catch (const std::bad_alloc&) {
    g_err = "out of host memory";
    return DUET_ENOMEM;
  } catch (const std::exception& e) {
    g_err = e.what();
    return DUET_EINVAL;
  } catch (...) {
    g_err = "unknown error";
    return DUET_EINVAL;
  }
}

template <class T>
void need(T* p, const char* what) {
  if (!p) fail(DUET_EINVAL, std::string(what) + " is NULL");
}
}  // namespace

extern "C" {

const char* duet_last_error(void) { return g_err.c_str(); }
int duet_abi_version(void) { return DUET_ABI_VERSION; }

duet_status duet_graph_load(const char* ir_text, size_t len, duet_graph_t** out) {
  if (out) *out = nullptr;
  return guard([&] {
    need(out, "out");
    need(ir_text, "ir_text");
    std::unique_ptr<duet_graph_t> h(new duet_graph_t());
    h->g.reset(parse_ir(ir_text, len));
    *out = h.release();
  });
}

duet_status duet_graph_bind(duet_graph_t* g, const char* param, const duet_tensor* t) {
  return guard([&] {
    need(g, "graph");
    need(param, "param");
    need(t, "tensor");
    auto it = g->g->params.find(param);
    if (it == g->g->params.end()) fail(DUET_EINVAL, std::string("no parameter @") + param);
    const ParamDecl& d = it->second;
    if ((int)t->dtype != d.dtype)
      fail(DUET_EDTYPE, std::string("@") + param + ": dtype " + dtype_name(t->dtype) + " != declared " +
                            dtype_name(d.dtype));
    if (t->ndim != (int)d.shape.size()) fail(DUET_ESHAPE, std::string("@") + param + ": rank mismatch");
    for (int i = 0; i < t->ndim; ++i)
      if (t->shape[i] != d.shape[i]) fail(DUET_ESHAPE, std::string("@") + param + ": shape mismatch");
    if (t->device < 0) fail(DUET_EINVAL, std::string("@") + param + ": parameters must be device memory");
    if (!t->data && d.numel() > 0) fail(DUET_EINVAL, std::string("@") + param + ": NULL data");
    for (auto& kv : g->g->bound)
      if (kv.second.device != t->device && kv.first != param)
        fail(DUET_EUNSUPPORTED, "all parameters must live on one GPU");
    g->g->bound[param] = Binding{t->data, t->device};
    g->g->prog.reset();  // weights changed: rebuild the device program lazily
  });
}

duet_status duet_graph_info(const duet_graph_t* g, int32_t* n_nodes, int32_t* n_inputs, int32_t* n_outputs,
                            int32_t* n_params) {
  return guard([&] {
    need(g, "graph");
    if (n_nodes) *n_nodes = (int32_t)g->g->nodes.size();
    if (n_inputs) *n_inputs = (int32_t)g->g->input_nodes.size();
    if (n_outputs) *n_outputs = (int32_t)g->g->outputs.size();
    if (n_params) *n_params = (int32_t)g->g->params.size();
  });
}

void duet_graph_destroy(duet_graph_t* g) { delete g; }

duet_status duet_partition(const duet_graph_t* g, const duet_partition_opts* o, duet_partition_t** out) {
  if (out) *out = nullptr;
  return guard([&] {
    need(g, "graph");
    need(out, "out");
    duet_partition_opts opts{0, 1};
    if (o) opts = *o;
    std::unique_ptr<duet_partition_t> h(new duet_partition_t());
    h->p.reset(make_partition(g->g.get(), opts.granularity, opts.batch_shards));
    *out = h.release();
  });
}

duet_status duet_partition_export(const duet_partition_t* p, int32_t* node_to_sg, int32_t* sg_phase,
                                  uint8_t* phase_kind, int32_t* edge_src, int32_t* edge_dst, int64_t* edge_bytes,
                                  int32_t* n_sg, int32_t* n_phase, int32_t* n_edge) {
  return guard([&] {
    need(p, "partition");
    const Partition& P = *p->p;
    if (n_sg) *n_sg = P.n_sg();
    if (n_phase) *n_phase = (int32_t)P.phase_kind.size();
    if (n_edge) *n_edge = (int32_t)P.edges.size();
    if (node_to_sg)
      for (size_t i = 0; i < P.node_to_sg.size(); ++i) node_to_sg[i] = P.node_to_sg[i];
    if (sg_phase)
      for (int s = 0; s < P.n_sg(); ++s) sg_phase[s] = P.sg_phase[s];
    if (phase_kind)
      for (size_t i = 0; i < P.phase_kind.size(); ++i) phase_kind[i] = (uint8_t)P.phase_kind[i];
    int k = 0;
    for (auto& kv : P.edges) {
      if (edge_src) edge_src[k] = kv.first.first;
      if (edge_dst) edge_dst[k] = kv.first.second;
      if (edge_bytes) edge_bytes[k] = kv.second;
      ++k;
    }
  });
}

duet_status duet_partition_shards(const duet_partition_t* p, int32_t* sg_shard, int32_t* sg_origin, int32_t* n_sg) {
  return guard([&] {
    need(p, "partition");
    const Partition& P = *p->p;
    if (n_sg) *n_sg = P.n_sg();
    for (int s = 0; s < P.n_sg(); ++s) {
      if (sg_shard) sg_shard[s] = P.sg_shard[s];
      if (sg_origin) sg_origin[s] = P.sg_origin[s];
    }
  });
}

void duet_partition_destroy(duet_partition_t* p) { delete p; }

static void no_shards(const Partition& P, const char* what) {
  if (P.sharded())
    fail(DUET_EUNSUPPORTED, std::string(what) +
                                ": a batch_shards > 1 partition is a scheduling model (its row shards run on "
                                "different ranks, multirank.ShardExecutor); profile it from a table");
}

duet_status duet_profile(const duet_partition_t* p, const duet_slot* slots, int n_slots, const duet_profile_opts* o,
                         duet_profile_t** out) {
  if (out) *out = nullptr;
  return guard([&] {
    need(p, "partition");
    need(out, "out");
    need(slots, "slots");
    if (n_slots < 1) fail(DUET_EINVAL, "n_slots < 1");
    no_shards(*p->p, "duet_profile");
    std::unique_ptr<duet_profile_t> h(new duet_profile_t());
    h->pr.reset(profile_on_device(p->p.get(), slots, n_slots, o));
    *out = h.release();
  });
}

duet_status duet_profile_from_table(const duet_partition_t* p, int n_slots, const int32_t* slot_gpu,
                                    const int64_t* t_ns, const duet_comm_model* c, duet_profile_t** out) {
  if (out) *out = nullptr;
  return guard([&] {
    need(p, "partition");
    need(out, "out");
    need(slot_gpu, "slot_gpu");
    need(t_ns, "t_ns");
    if (n_slots < 1) fail(DUET_EINVAL, "n_slots < 1");
    std::unique_ptr<Profile> pr(new Profile());
    pr->p = p->p.get();
    pr->n_slots = n_slots;
    pr->slot_gpu.assign(slot_gpu, slot_gpu + n_slots);
    size_t n = (size_t)p->p->n_sg() * n_slots;
    pr->t_ns.assign(t_ns, t_ns + n);
    for (auto v : pr->t_ns)
      if (v < 0) fail(DUET_EINVAL, "negative time in profile table");
    if (c) pr->comm = *c;
    if (pr->comm.same_gpu.alpha_ns < 0 || pr->comm.cross_gpu.alpha_ns < 0 || pr->comm.same_gpu.ps_per_byte < 0 ||
        pr->comm.cross_gpu.ps_per_byte < 0)
      fail(DUET_EINVAL, "negative comm model");
    std::unique_ptr<duet_profile_t> h(new duet_profile_t());
    h->pr = std::move(pr);
    *out = h.release();
  });
}

duet_status duet_profile_export(const duet_profile_t* pr, int64_t* t_ns, int32_t* slot_gpu, duet_comm_model* c,
                                int32_t* n_slots) {
  return guard([&] {
    need(pr, "profile");
    const Profile& P = *pr->pr;
    if (n_slots) *n_slots = P.n_slots;
    if (t_ns) memcpy(t_ns, P.t_ns.data(), P.t_ns.size() * sizeof(int64_t));
    if (slot_gpu)
      for (int d = 0; d < P.n_slots; ++d) slot_gpu[d] = P.slot_gpu[d];
    if (c) *c = P.comm;
  });
}

void duet_profile_destroy(duet_profile_t* pr) { delete pr; }

duet_status duet_schedule(const duet_partition_t* p, const duet_profile_t* pr, const duet_sched_opts* o,
                          duet_schedule_t** out) {
  if (out) *out = nullptr;
  return guard([&] {
    need(p, "partition");
    need(pr, "profile");
    need(out, "out");
    std::unique_ptr<duet_schedule_t> h(new duet_schedule_t());
    h->s.reset(make_schedule(p->p.get(), pr->pr.get(), o));
    *out = h.release();
  });
}

duet_status duet_schedule_measured(const duet_partition_t* p, const duet_profile_t* pr, const duet_sched_opts* o,
                                   const duet_slot* slots, int n_slots, duet_measure_opts* mo, duet_schedule_t** out) {
  if (out) *out = nullptr;
  return guard([&] {
    need(p, "partition");
    need(pr, "profile");
    need(slots, "slots");
    need(out, "out");
    no_shards(*p->p, "duet_schedule_measured");
    std::unique_ptr<duet_schedule_t> h(new duet_schedule_t());
    h->s.reset(schedule_measured(p->p.get(), pr->pr.get(), o, slots, n_slots, mo));
    *out = h.release();
  });
}

duet_status duet_schedule_export(const duet_schedule_t* s, int32_t* sg_to_slot, int32_t* order,
                                 int64_t* model_makespan_ns, int32_t* fell_back) {
  return guard([&] {
    need(s, "schedule");
    const Schedule& S = *s->s;
    for (size_t i = 0; i < S.slot_of.size(); ++i) {
      if (sg_to_slot) sg_to_slot[i] = S.slot_of[i];
      if (order) order[i] = S.order[i];
    }
    if (model_makespan_ns) *model_makespan_ns = S.makespan;
    if (fell_back) *fell_back = S.fell_back;
  });
}

void duet_schedule_destroy(duet_schedule_t* s) { delete s; }

duet_status duet_run(duet_schedule_t* s, const duet_slot* slots, int n_slots, const duet_tensor* inputs, int n_in,
                     duet_tensor* outputs, int n_out) {
  return guard([&] {
    need(s, "schedule");
    need(slots, "slots");
    if (n_in && !inputs) fail(DUET_EINVAL, "inputs is NULL");
    if (n_out && !outputs) fail(DUET_EINVAL, "outputs is NULL");
    no_shards(*s->s->p, "duet_run");
    run_schedule(s->s.get(), slots, n_slots, inputs, n_in, outputs, n_out);
  });
}

duet_status duet_schedule_set_trace(duet_schedule_t* s, int on) {
  return guard([&] {
    need(s, "schedule");
    s->s->trace = on ? 1 : 0;
  });
}

duet_status duet_schedule_trace(const duet_schedule_t* s, int64_t* start_ns, int64_t* end_ns, int32_t n_sg) {
  return guard([&] {
    need(s, "schedule");
    schedule_trace_export(s->s.get(), start_ns, end_ns, n_sg);
  });
}

duet_status duet_schedule_launch_count(const duet_schedule_t* s, int64_t* n_kernels) {
  return guard([&] {
    need(s, "schedule");
    need(n_kernels, "n_kernels");
    *n_kernels = schedule_launch_count(s->s.get());
  });
}

duet_status duet_node_run(duet_graph_t* g, const char* node_name, const duet_tensor* args, int n_args,
                          duet_tensor* out, void* stream) {
  return guard([&] {
    need(g, "graph");
    need(node_name, "node_name");
    need(out, "out");
    node_run(g->g.get(), node_name, args, n_args, out, stream);
  });
}

}  // extern "C"
