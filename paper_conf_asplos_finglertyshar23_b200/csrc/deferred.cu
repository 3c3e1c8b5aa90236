// deferred.cu — memory release that never blocks behind a persistent server kernel.
//
// cudaFree and cudaFreeHost wait until the device is idle, and a persistent doorbell server
// (server.cu, NEXT-2) keeps a kernel resident until lake_linnos_server_stop. A free issued
// while any server runs would therefore hang the caller (and with it the server's client).
// Every release in the library goes through release_device / release_host: immediate when
// no server runs (on any device: pinned host memory is portable, so its release is
// conservatively treated as process-wide), otherwise parked until the last server stops.
#include <cuda_runtime.h>

#include <mutex>
#include <new>

#include "lake_internal.h"

namespace lake {
namespace {

struct Parked {
  void *p;
  int device;  // -1: pinned host memory
  Parked *next;
};

std::mutex g_mu;
int g_servers = 0;
Parked *g_parked = nullptr;

void free_now(void *p, int device) {
  if (device < 0) {
    cudaFreeHost(p);
    return;
  }
  int prev = -1;
  cudaGetDevice(&prev);
  if (prev != device) cudaSetDevice(device);
  cudaFree(p);
  if (prev >= 0 && prev != device) cudaSetDevice(prev);
}

void release(void *p, int device) {
  if (!p) return;
  std::lock_guard<std::mutex> lk(g_mu);
  if (g_servers == 0) {
    free_now(p, device);
    return;
  }
  Parked *e = new (std::nothrow) Parked{p, device, g_parked};
  if (e) g_parked = e;  // out of host memory: leak rather than block behind a server
}

}  // namespace

void release_device(void *p, int device) { release(p, device); }
void release_host(void *p) { release(p, -1); }

void servers_started() {
  std::lock_guard<std::mutex> lk(g_mu);
  ++g_servers;
}

void servers_stopped() {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g_servers > 0) --g_servers;
  if (g_servers > 0) return;
  while (g_parked) {
    Parked *e = g_parked;
    g_parked = e->next;
    free_now(e->p, e->device);
    delete e;
  }
}

}  // namespace lake
