// NCCL communicator behind crsd_comm_t (dist.cpp, solver.cpp).
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>

struct crsd_comm_s {
    ncclComm_t comm = nullptr;
    int rank = 0, world = 1, device = 0;
    cudaStream_t cs = nullptr;                         // halo exchange stream
    cudaEvent_t ev_x = nullptr, ev_halo = nullptr;
};
