// mgpu.h — internal interface of the multi-GPU executor (mgpu.cu; not part of the C-ABI).
//
// a cube sharded block-cyclically on dimension 0 is answered by every
// shard reducing its part of each query into per-query partials (a3-a7), ONE exchange of those
// partials over NCCL (sum with +, MIN/MAX codes with max; 16 B per query), and the finalize
// (a9).  An Exec runs that path for one cube handle:
//   * a group handle (olap_cube_create_multi): G = ndevices x shards_per_device shards in this
//     process, one NCCL communicator per device (ncclCommInitAll), ncclReduce to devices[0];
//   * a shard with an attached communicator (olap_cube_attach_comm; one process per GPU):
//     ncclAllReduce, so every rank finalizes every answer;
//   * a plain cube (olap_query_stream only): no exchange.
// Batches are issued on internal per-device streams: a compute stream (inputs, partials, local
// combine) and an exchange stream (NCCL, finalize, results), with ping-pong buffers, so batch
// k's exchange and finalize overlap batch k+1's range-reduce (olap_query_stream).
#pragma once

#include <vector>

#include "common.cuh"

namespace olap {

struct Exec;
struct Group;

// every shard / device of an Exec; `shards[i]` lives on `devices[i / spd]`
struct ExecSpec {
    int nd = 0, dtype = 0;
    int64_t n[8] = {};
    std::vector<int> devices;
    std::vector<olap_cube*> shards;  // borrowed
    int spd = 1;                     // shards per device
    olap_comm* comm = nullptr;       // multi-process communicator (borrowed), or
    bool own_comms = false;          // group: one communicator per device (ncclCommInitAll)
};

int exec_create(const ExecSpec& spec, Exec** out);
void exec_destroy(Exec* e);
int exec_query_batch(Exec* e, int64_t nq, const olap_range* ranges, const int32_t* ops, olap_result* results);
int exec_query_batch_device(Exec* e, int64_t nq, const olap_range* d_ranges, const int32_t* d_ops,
                            olap_result* d_results, cudaStream_t st);
int exec_query_stream(Exec* e, int64_t nq, const olap_range* ranges, const int32_t* ops, olap_result* results,
                      int64_t batch);
int64_t exec_launches(const Exec* e);  // combine kernels the executor launched (finalize: olap_finalize_launches)

// host-side validation shared by the host-buffer entry points (OLAP_E_RANGE names the query)
int validate_queries(int nd, const int64_t* n, int64_t nq, const olap_range* ranges, const int32_t* ops);

}  // namespace olap
