// comm.cuh -- the collective the sharded driver needs, behind one
// small interface so the same level loop runs over NCCL (one process per GPU,
// NVLink/NVSwitch) or over an in-process group of contexts (virtual ranks
// for tests, every rank a host thread).
//
// The sharded level loop exchanges exactly one kind of message: a buffer in
// which every rank fills a disjoint set of slots and leaves the rest zero, and
// which every rank needs in full -- the level's sample keys (each rank owns a
// range of sample slots), the per-rank counts of the level (rank r owns row r),
// and the gathered survivors (rank r owns a range of positions).  An integer
// sum-allreduce over such a buffer is an allgather with the ranks' placement
// decided on the device (the offsets never pass through the host), and it is
// exact: every slot is x + 0 + ... + 0.  Keys and raw element bits are summed
// as u32 / u64 integers.
#pragma once
#include <string>
#include <cuda_runtime.h>
#include "sampleselect.h"

struct ss_local_group;   // opaque, include/sampleselect.h

namespace ss_comm {

class ShardComm {
public:
    virtual ~ShardComm() {}
    virtual int nranks() const = 0;
    virtual int rank() const = 0;
    // may be captured into a CUDA graph (host-synchronising groups may not)
    virtual bool capturable() const = 0;
    // recv[i] = sum over ranks of send[i] (u32 or u64 wrap-around, elem_bytes 4
    // or 8), enqueued on `st`; send == recv is allowed
    virtual ss_status allreduce_sum(const void* send, void* recv, size_t count, int elem_bytes, cudaStream_t st,
                                    std::string& err) = 0;
};

// NCCL (resolved at run time with dlopen: the library loads without NCCL)
ss_status nccl_unique_id(char out[128], std::string& err);
ShardComm* make_nccl_comm(const char id[128], int nranks, int rank, int device, ss_status* rc, std::string& err);
// in-process group
ss_status local_group_create(int nranks, ss_local_group** out);
void local_group_destroy(ss_local_group* g);
ShardComm* make_local_comm(ss_local_group* g, int rank, int device, ss_status* rc, std::string& err);

}  // namespace ss_comm
