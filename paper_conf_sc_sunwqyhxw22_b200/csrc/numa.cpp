// NUMA placement of the pinned host store and of the CPU Adam workers (SURVEY §8(a) a1:
// "Pinned NUMA-aware host store ... Placement SPLIT (layer k -> node k mod n; Adam threads of
// that node) or LOCAL (GPU's node); DP: slice r of every layer on GPU r's node").
//
// The paper pins one buffer per layer in CPU RAM and runs several concurrent
// optimizers on the multi-core host (its box is a 2-socket Xeon).  On a
// multi-socket host the CPU Adam is bound by local DRAM bandwidth, so where a layer's master /
// m / v live and which cores update it decides whether the update streams from local or remote
// memory.  There are no libnuma headers in the image, so this file talks to the kernel directly:
// topology from sysfs, placement with the mbind(2) syscall before the first touch, worker
// affinity with pthread_setaffinity_np.  On a single-node host every call is a no-op.
//
// SH_SYSFS_ROOT (tests only) prefixes every sysfs path, so the topology parser and the policy
// plan can be exercised with a fake multi-node tree on a one-node machine.
#include <pthread.h>
#include <sys/mman.h>
#include <sched.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <algorithm>
#include <cctype>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "sh_internal.hpp"

namespace sh {
namespace numa {

namespace {
// <linux/mempolicy.h> values (stable kernel ABI)
constexpr int kMpolPreferred = 1;
constexpr int kMpolBind = 2;
constexpr int kMpolInterleave = 3;
constexpr unsigned kMpolMfMove = 1u << 1;
constexpr int kMpolFNode = 1 << 0;
constexpr int kMpolFAddr = 1 << 1;
constexpr int kMaxNodes = 1024;

std::string sysfs_root() {
  const char* r = getenv("SH_SYSFS_ROOT");
  return r ? std::string(r) : std::string();
}

bool read_line(const std::string& path, std::string* out) {
  FILE* f = fopen(path.c_str(), "r");
  if (!f) return false;
  char buf[8192];
  const bool ok = fgets(buf, sizeof(buf), f) != nullptr;
  fclose(f);
  if (!ok) return false;
  *out = buf;
  while (!out->empty() && isspace((unsigned char)out->back())) out->pop_back();
  return true;
}

std::mutex g_mu;
Topology g_topo;
bool g_topo_done = false;
}  // namespace

// "0-3,8,10-11" -> {0,1,2,3,8,10,11}.  Returns false on a malformed list.
bool parse_cpulist(const char* s, std::vector<int>* out) {
  out->clear();
  const char* p = s;
  while (*p) {
    while (*p == ',' || isspace((unsigned char)*p)) ++p;
    if (!*p) break;
    if (!isdigit((unsigned char)*p)) return false;
    char* e = nullptr;
    const long a = strtol(p, &e, 10);
    long b = a;
    p = e;
    if (*p == '-') {
      ++p;
      if (!isdigit((unsigned char)*p)) return false;
      b = strtol(p, &e, 10);
      p = e;
    }
    if (b < a || b > 1 << 20) return false;
    for (long c = a; c <= b; ++c) out->push_back((int)c);
    if (*p && *p != ',' && !isspace((unsigned char)*p)) return false;
  }
  return true;
}

Topology read_topology() {
  Topology t;
  const std::string root = sysfs_root() + "/sys/devices/system/node";
  std::string online;
  std::vector<int> ids;
  if (read_line(root + "/online", &online) && parse_cpulist(online.c_str(), &ids)) {
    for (int id : ids) {
      if (id < 0 || id >= kMaxNodes) continue;
      std::string cl;
      std::vector<int> cpus;
      if (!read_line(root + "/node" + std::to_string(id) + "/cpulist", &cl) || !parse_cpulist(cl.c_str(), &cpus))
        cpus.clear();
      t.node_ids.push_back(id);
      t.cpus.push_back(cpus);
    }
  }
  if (t.node_ids.empty()) {  // no NUMA sysfs: one node holding every online CPU
    t.node_ids.push_back(0);
    std::vector<int> all;
    const long n = sysconf(_SC_NPROCESSORS_ONLN);
    for (long c = 0; c < std::max(1L, n); ++c) all.push_back((int)c);
    t.cpus.push_back(all);
  }
  return t;
}

const Topology& topology() {
  std::lock_guard<std::mutex> g(g_mu);
  if (!g_topo_done) {
    g_topo = read_topology();
    g_topo_done = true;
  }
  return g_topo;
}

void reset_topology_cache() {
  std::lock_guard<std::mutex> g(g_mu);
  g_topo_done = false;
}

// Index (into topology().node_ids) of the node a PCI device hangs off; 0 when unknown.
int node_index_of_pci(const char* bus_id) {
  const Topology& t = topology();
  std::string id(bus_id ? bus_id : "");
  for (auto& ch : id) ch = (char)tolower((unsigned char)ch);
  std::string v;
  // cudaDeviceGetPCIBusId gives "0000:1b:00.0"; sysfs uses the same form in lower case
  if (id.empty() || !read_line(sysfs_root() + "/sys/bus/pci/devices/" + id + "/numa_node", &v)) return 0;
  const int node = atoi(v.c_str());
  for (size_t k = 0; k < t.node_ids.size(); ++k)
    if (t.node_ids[k] == node) return (int)k;
  return 0;  // -1 ("no affinity") or an offline node
}

int gpu_node_index(int device) {
  char bus[64] = {0};
  if (cudaDeviceGetPCIBusId(bus, sizeof(bus), device) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return node_index_of_pci(bus);
}

int resolve_policy(int policy, int n_nodes, bool shared) {
  if (policy == SH_NUMA_AUTO) {
    if (n_nodes <= 1) return SH_NUMA_NONE;
    return shared ? SH_NUMA_LOCAL : SH_NUMA_SPLIT;
  }
  return policy;
}

// Placement target of host-store unit `unit` (a layer; with a shared store the unit is a rank's
// slice and the caller passes that rank's GPU node as gpu_node with policy LOCAL).
// Returns a node INDEX >= 0, kInterleave, or kNone.
int plan_node(int policy, int unit, int n_nodes, int gpu_node) {
  if (n_nodes <= 1) return kNone;
  switch (policy) {
    case SH_NUMA_SPLIT: return ((unit % n_nodes) + n_nodes) % n_nodes;
    case SH_NUMA_LOCAL: return std::min(std::max(gpu_node, 0), n_nodes - 1);
    case SH_NUMA_INTERLEAVE: return kInterleave;
    default: return kNone;
  }
}

// Node index a CPU Adam worker is pinned to (kNone: not pinned).  SPLIT spreads the workers
// over the nodes in proportion to their core counts (round robin over the nodes' cores), LOCAL
// pins all of them to the GPU's node.
int worker_node(int policy, int tid, int n_threads, int gpu_node) {
  const Topology& t = topology();
  const int n = (int)t.node_ids.size();
  if (n <= 1) return kNone;
  if (policy == SH_NUMA_LOCAL) return std::min(std::max(gpu_node, 0), n - 1);
  if (policy != SH_NUMA_SPLIT) return kNone;
  // core list in node-interleaved order: node0 cpu0, node1 cpu0, node0 cpu1, ...
  std::vector<int> order;
  size_t most = 0;
  for (auto& c : t.cpus) most = std::max(most, c.size());
  for (size_t i = 0; i < most; ++i)
    for (int k = 0; k < n; ++k)
      if (i < t.cpus[k].size()) order.push_back(k);
  if (order.empty()) return tid % n;
  (void)n_threads;
  return order[tid % order.size()];
}

bool bind_range(void* p, size_t bytes, int node_index) {
  if (node_index == kNone || !p || bytes == 0) return true;
  const Topology& t = topology();
  const long page = sysconf(_SC_PAGESIZE);
  uintptr_t a = reinterpret_cast<uintptr_t>(p);
  uintptr_t e = a + bytes;
  a = (a + page - 1) / page * page;  // pages wholly inside the range
  e = e / page * page;
  if (e <= a) return true;
  std::vector<unsigned long> mask(kMaxNodes / (8 * sizeof(unsigned long)), 0ul);
  int mode;
  if (node_index == kInterleave) {
    mode = kMpolInterleave;
    for (int id : t.node_ids) mask[id / (8 * sizeof(unsigned long))] |= 1ul << (id % (8 * sizeof(unsigned long)));
  } else {
    if (node_index < 0 || node_index >= (int)t.node_ids.size()) return false;
    const int id = t.node_ids[node_index];
    // PREFERRED: the node's pages when it has them, any node when it runs out (never an OOM
    // kill for a full node; the pinned store already checks MemAvailable)
    mode = kMpolPreferred;
    mask[id / (8 * sizeof(unsigned long))] |= 1ul << (id % (8 * sizeof(unsigned long)));
  }
  const long r = syscall(SYS_mbind, (void*)a, (unsigned long)(e - a), mode, mask.data(),
                         (unsigned long)kMaxNodes + 1, kMpolMfMove);
  return r == 0;
}

bool bind_strict(void* p, size_t bytes, int node_id) {
  std::vector<unsigned long> mask(kMaxNodes / (8 * sizeof(unsigned long)), 0ul);
  mask[node_id / (8 * sizeof(unsigned long))] |= 1ul << (node_id % (8 * sizeof(unsigned long)));
  return syscall(SYS_mbind, p, (unsigned long)bytes, kMpolBind, mask.data(), (unsigned long)kMaxNodes + 1,
                 kMpolMfMove) == 0;
}

int node_of_page(const void* p) {
  int node = -1;
  const long r = syscall(SYS_get_mempolicy, &node, nullptr, 0ul, const_cast<void*>(p), kMpolFNode | kMpolFAddr);
  return r == 0 ? node : -1;
}

bool pin_thread(int node_index) {
  if (node_index == kNone) return true;
  const Topology& t = topology();
  if (node_index < 0 || node_index >= (int)t.cpus.size() || t.cpus[node_index].empty()) return false;
  cpu_set_t set;
  CPU_ZERO(&set);
  for (int c : t.cpus[node_index])
    if (c < CPU_SETSIZE) CPU_SET(c, &set);
  return pthread_setaffinity_np(pthread_self(), sizeof(set), &set) == 0;
}

}  // namespace numa
}  // namespace sh

using namespace sh;

extern "C" {

int32_t sh_numa_topology(int32_t* node_ids, int32_t* n_cpus, int32_t cap) {
  numa::reset_topology_cache();  // re-read (tests switch SH_SYSFS_ROOT)
  const numa::Topology& t = numa::topology();
  const int n = (int)t.node_ids.size();
  for (int k = 0; k < n && k < cap; ++k) {
    if (node_ids) node_ids[k] = t.node_ids[k];
    if (n_cpus) n_cpus[k] = (int32_t)t.cpus[k].size();
  }
  return n;
}

int32_t sh_numa_plan(int32_t policy, int32_t unit, int32_t n_nodes, int32_t gpu_node, int32_t shared) {
  return numa::plan_node(numa::resolve_policy(policy, n_nodes, shared != 0), unit, n_nodes, gpu_node);
}

int32_t sh_numa_worker_node(int32_t policy, int32_t tid, int32_t n_threads, int32_t gpu_node) {
  numa::reset_topology_cache();
  const int n = (int)numa::topology().node_ids.size();
  return numa::worker_node(numa::resolve_policy(policy, n, false), tid, n_threads, gpu_node);
}

int32_t sh_numa_node_of_pci(const char* bus_id) {
  numa::reset_topology_cache();
  return numa::node_index_of_pci(bus_id);
}

int32_t sh_numa_bind_check(int32_t node_id, int64_t bytes) {
  // mbind(MPOL_BIND) an anonymous mapping to node_id, touch it, and return the node
  // get_mempolicy reports for its first and last page (-1 on failure)
  if (bytes <= 0) return -1;
  void* p = mmap(nullptr, (size_t)bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  if (p == MAP_FAILED) return -1;
  int r = -1;
  if (numa::bind_strict(p, (size_t)bytes, node_id)) {
    memset(p, 1, (size_t)bytes);
    const long page = sysconf(_SC_PAGESIZE);
    const int a = numa::node_of_page(p);
    const int b = numa::node_of_page(static_cast<char*>(p) + ((bytes - 1) / page) * page);
    r = (a == b) ? a : -1;
  }
  munmap(p, (size_t)bytes);
  return r;
}

}  // extern "C"
