// baselines.cu — the CPU-controlled comparison modes (Listing 2.1a, P:528-531,
// SURVEY §8(a) a10 and §8(f) N1): per-iteration host launches + halo copies / NCCL / NVSHMEM,
// and the CUDA-graph-captured loop.
#include "runtime_internal.h"

namespace jbrt {
int ensure_nccl(jacobi_ctx *h) {
  if (h->nccl_ready) return JACOBI_OK;
  if (h->kind == KIND_VIRTUAL && h->total > 1) return JACOBI_EINVAL;  // NCCL: one rank per GPU
  if (h->kind == KIND_DIST) return JACOBI_ESTATE;  // needs jacobi_nccl_init via the binding
  if (h->kind == KIND_SHMEM) return JACOBI_EINVAL;
  if (!g_nccl.load()) return JACOBI_ENCCL;
  std::vector<int> devs;
  for (auto &s : h->slabs) devs.push_back(s.device);
  std::vector<ncclComm_t> comms(devs.size());
  if (g_nccl.CommInitAll(comms.data(), (int)devs.size(), devs.data()) != ncclSuccess) return JACOBI_ENCCL;
  for (size_t i = 0; i < devs.size(); ++i) h->slabs[i].comm = comms[i];
  h->nccl_ready = true;
  return JACOBI_OK;
}

// CPU-controlled baselines (Listing 2.1a).
// Every iteration the host launches discrete kernels on every GPU, moves the edge planes into
// the neighbours' halos, and synchronises every GPU before the next iteration (the
// OpenMP/MPI barrier of the reference code):
//   COPY    : kernel over all planes, then cudaMemcpyPeerAsync of the edge planes
//   NCCL    : kernel, then ncclSend/ncclRecv of the edge planes (grouped)
//   OVERLAP : boundary planes on a comm stream (few CTAs) + memcpy, interior planes concurrently
//             on the compute stream ("Baseline Overlap")
//   P2P     : one kernel whose boundary CTAs store the edge planes into the peers' halos
//   GRAPH   : the COPY loop captured once into a CUDA graph (all iterations, cross-GPU event
//             dependencies instead of host barriers) and replayed with one launch — the strongest
//             CPU-controlled variant (not in the paper).


int time_begin(jacobi_ctx *h) {
  for (auto &s : h->slabs) {
    CK(cudaSetDevice(s.device));
    CK(reset_run_counters(s, s.stream));
    CK(cudaEventRecord(s.ev0, s.stream));
  }
  return JACOBI_OK;
}

int time_end(jacobi_ctx *h, int64_t iters) {
  double mx = 0;
  for (auto &s : h->slabs) {
    CK(cudaSetDevice(s.device));
    CK(cudaEventRecord(s.ev1, s.stream));
    CK(cudaEventSynchronize(s.ev1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, s.ev0, s.ev1));
    s.last_ms = ms;
    mx = std::max(mx, (double)ms);
  }
  h->last_ms_max = mx;
  h->t += iters;
  // Keep the CPU-Free protocol consistent: inbound flags hold the global iteration count.
  for (auto &s : h->slabs) {
    CK(cudaSetDevice(s.device));
    CK(jbk::launch_flag_max(&s.ctrl->flag_in[0][0], 2 * JB_MAXK, (unsigned long long)h->t, s.stream));
    ++h->last_launches;
    CK(cudaStreamSynchronize(s.stream));
  }
  return JACOBI_OK;
}

// Host-issued peer copies of slab s's edge planes of buffer `nxt` into its neighbours' halos.
// (Inside a graph capture the UVA form cudaMemcpyAsync(cudaMemcpyDefault) is used: it is the
// capturable equivalent of cudaMemcpyPeerAsync once peer access is enabled.)
int copy_edges(jacobi_ctx *h, Slab &s, int nxt, cudaStream_t st, bool capturing) {
  const int64_t pe = h->geom.plane_elems;
  const size_t bytes = (size_t)pe * sizeof(double);
  if (capturing) {
    if (s.has_top) CK(cudaMemcpyAsync(s.peer_top[nxt], s.buf[nxt] + 1 * pe, bytes, cudaMemcpyDefault, st));
    if (s.has_bot) CK(cudaMemcpyAsync(s.peer_bot[nxt], s.buf[nxt] + s.chunk * pe, bytes, cudaMemcpyDefault, st));
    return JACOBI_OK;
  }
  if (s.has_top)
    CK(cudaMemcpyPeerAsync(s.peer_top[nxt], s.peer_top_dev, s.buf[nxt] + 1 * pe, s.device, bytes, st));
  if (s.has_bot)
    CK(cudaMemcpyPeerAsync(s.peer_bot[nxt], s.peer_bot_dev, s.buf[nxt] + s.chunk * pe, s.device, bytes, st));
  return JACOBI_OK;
}

int nccl_edges(jacobi_ctx *h, int nxt) {
  const int64_t pe = h->geom.plane_elems;
  if (g_nccl.GroupStart() != ncclSuccess) return JACOBI_ENCCL;
  for (auto &s : h->slabs) {
    const int me = s.id;
    double *b = s.buf[nxt];
    if (s.has_top) {
      if (g_nccl.Send(b + 1 * pe, pe, ncclFloat64, me - 1, s.comm, s.stream) != ncclSuccess) return JACOBI_ENCCL;
      if (g_nccl.Recv(b, pe, ncclFloat64, me - 1, s.comm, s.stream) != ncclSuccess) return JACOBI_ENCCL;
    }
    if (s.has_bot) {
      if (g_nccl.Send(b + s.chunk * pe, pe, ncclFloat64, me + 1, s.comm, s.stream) != ncclSuccess)
        return JACOBI_ENCCL;
      if (g_nccl.Recv(b + (s.chunk + 1) * pe, pe, ncclFloat64, me + 1, s.comm, s.stream) != ncclSuccess)
        return JACOBI_ENCCL;
    }
  }
  if (g_nccl.GroupEnd() != ncclSuccess) return JACOBI_ENCCL;
  return JACOBI_OK;
}

int run_graph(jacobi_ctx *h, int64_t iters, bool nocomp, std::vector<LaunchPlan> &plans);

int run_baseline(jacobi_ctx *h, int64_t iters, BaseKind kind) {
  h->last_launches = 0;
  const bool nocomp = h->flags & JACOBI_FLAG_NO_COMPUTE;
  if (kind == BK_NCCL) {
    int rc = ensure_nccl(h);
    if (rc) return rc;
  } else if (kind == BK_SHMEM) {
    if (h->kind != KIND_SHMEM) return JACOBI_EINVAL;  // needs the NVSHMEM variant's handles
  } else if ((h->kind == KIND_DIST || h->kind == KIND_SHMEM) && h->total > 1) {
    return JACOBI_EINVAL;  // host-synchronised peer baselines need one process: use NCCL
  }
  const int n = (int)h->slabs.size();
  std::vector<LaunchPlan> plans(n), edges(n);
  for (int i = 0; i < n; ++i) {
    Slab &s = h->slabs[i];
    int rc;
    if (kind == BK_P2P || kind == BK_SHMEM) {
      rc = plan_launch(h, {i}, LK_P2P, nocomp, plans[i]);
    } else if (kind == BK_OVERLAP && (s.has_top || s.has_bot)) {
      int sms = 0;
      CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, s.device));
      const int ne = std::max(2, std::min(sms / 8, 32));  // boundary CTAs on the comm stream
      rc = plan_launch(h, {i}, LK_EDGES, nocomp, edges[i], ne);
      if (!rc) rc = plan_launch(h, {i}, LK_INNER, nocomp, plans[i], sms - edges[i].grid);
    } else {
      rc = plan_launch(h, {i}, LK_ALL, nocomp, plans[i]);
    }
    if (rc) return rc;
    plans[i].P.iters = 1;
    edges[i].P.iters = 1;
  }
  if (kind == BK_GRAPH) return run_graph(h, iters, nocomp, plans);
  int rc = time_begin(h);
  if (rc) return rc;
  // P2P / NVSHMEM no-compute still move halos in-kernel
  const bool launch_kernels = !nocomp || kind == BK_P2P || kind == BK_SHMEM;
  for (int64_t it = 0; it < iters; ++it) {
    const int64_t tg = h->t + it;
    const int nxt = (int)((tg + 1) & 1);
    for (int i = 0; i < n; ++i) {  // ② launch the kernel(s) on every GPU
      Slab &s = h->slabs[i];
      CK(cudaSetDevice(s.device));
      if (kind == BK_OVERLAP && edges[i].grid > 0) {
        // comm stream: boundary planes first, then the peer copies; compute stream: interior
        if (!nocomp) {
          edges[i].P.t0 = tg;
          CK(jbk::launch_sweep(edges[i].P, false, false, edges[i].grid, edges[i].smem, s.stream2));
          ++h->last_launches;
          plans[i].P.t0 = tg;
          CK(jbk::launch_sweep(plans[i].P, false, false, plans[i].grid, plans[i].smem, s.stream));
          ++h->last_launches;
        }
        rc = copy_edges(h, s, nxt, s.stream2);
        if (rc) return rc;
        continue;
      }
      if (launch_kernels) {
        plans[i].P.t0 = tg;
        CK(jbk::launch_sweep(plans[i].P, nocomp, false, plans[i].grid, plans[i].smem, s.stream));
        ++h->last_launches;
      }
    }
    if (kind == BK_COPY) {  // ④ write_neighbors with host-issued peer copies
      for (auto &s : h->slabs) {
        CK(cudaSetDevice(s.device));
        rc = copy_edges(h, s, nxt, s.stream);
        if (rc) return rc;
      }
    } else if (kind == BK_NCCL) {
      rc = nccl_edges(h, nxt);
      if (rc) return rc;
    } else if (kind == BK_SHMEM) {
      // the second per-iteration kernel waits for the neighbours' signals; no host
      // barrier — the next iteration's kernel is ordered behind it on the stream.
      for (int i = 0; i < n; ++i) {
        Slab &s = h->slabs[i];
        CK(cudaSetDevice(s.device));
        CK(jbk::launch_neighbour_wait(plans[i].P, (unsigned long long)(tg + 1), s.stream));
        ++h->last_launches;
      }
      continue;
    }
    for (auto &s : h->slabs) {  // ⑤ sync streams, host barrier: wait for every GPU
      CK(cudaSetDevice(s.device));
      CK(cudaStreamSynchronize(s.stream2));
      CK(cudaStreamSynchronize(s.stream));
    }
  }
  return time_end(h, iters);
}

// GRAPH baseline: capture `iters` iterations of (kernel; peer copies) for every slab into one
// graph.  Slab g's kernel of iteration t+1 waits (graph edge) for the copies of its neighbours
// at iteration t; its copies follow its own kernel.  The instantiated graph is cached per
// (iters, parity of t, plan generation).
int run_graph(jacobi_ctx *h, int64_t iters, bool nocomp, std::vector<LaunchPlan> &plans) {
  const int n = (int)h->slabs.size();
  const int parity = (int)(h->t & 1);
  if (!h->graph_exec || h->graph_iters != iters || h->graph_parity != parity || h->graph_gen != h->plan_gen) {
    if (h->graph_exec) cudaGraphExecDestroy(h->graph_exec);
    h->graph_exec = nullptr;
    Slab &m = h->slabs[0];
    CK(cudaSetDevice(m.device));
    CK(cudaStreamBeginCapture(m.stream, cudaStreamCaptureModeRelaxed));
    CK(cudaEventRecord(m.ev_sync, m.stream));
    for (int i = 1; i < n; ++i) {  // fork every other slab's stream into the capture
      CK(cudaSetDevice(h->slabs[i].device));
      CK(cudaStreamWaitEvent(h->slabs[i].stream, m.ev_sync, 0));
    }
    for (int64_t it = 0; it < iters; ++it) {
      const int64_t tg = h->t + it;
      const int nxt = (int)((tg + 1) & 1);
      for (int i = 0; i < n; ++i) {
        Slab &s = h->slabs[i];
        CK(cudaSetDevice(s.device));
        if (it > 0) {  // halos of this iteration were written by the neighbours' copies
          if (s.has_top) CK(cudaStreamWaitEvent(s.stream, h->slabs[i - 1].ev_copy, 0));
          if (s.has_bot) CK(cudaStreamWaitEvent(s.stream, h->slabs[i + 1].ev_copy, 0));
        }
        if (!nocomp) {
          plans[i].P.t0 = tg;
          CK(jbk::launch_sweep(plans[i].P, false, false, plans[i].grid, plans[i].smem, s.stream));
        }
      }
      for (int i = 0; i < n; ++i) {
        Slab &s = h->slabs[i];
        CK(cudaSetDevice(s.device));
        int rc = copy_edges(h, s, nxt, s.stream, true);
        if (rc) {
          cudaGraph_t g;
          cudaStreamEndCapture(m.stream, &g);
          return rc;
        }
        CK(cudaEventRecord(s.ev_copy, s.stream));
      }
    }
    CK(cudaSetDevice(m.device));
    for (int i = 1; i < n; ++i) CK(cudaStreamWaitEvent(m.stream, h->slabs[i].ev_copy, 0));  // join
    cudaGraph_t graph;
    CK(cudaStreamEndCapture(m.stream, &graph));
    cudaError_t e = cudaGraphInstantiate(&h->graph_exec, graph, 0);
    cudaGraphDestroy(graph);
    CK(e);
    h->graph_iters = iters;
    h->graph_parity = parity;
    h->graph_gen = h->plan_gen;
  }
  int rc = time_begin(h);
  if (rc) return rc;
  Slab &m = h->slabs[0];
  CK(cudaSetDevice(m.device));
  CK(cudaGraphLaunch(h->graph_exec, m.stream));
  h->last_launches += nocomp ? 0 : iters * n;  // the graph's kernel nodes
  CK(cudaStreamSynchronize(m.stream));
  return time_end(h, iters);
}
}  // namespace jbrt
