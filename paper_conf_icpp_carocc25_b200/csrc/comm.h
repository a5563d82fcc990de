// comm.h — host side of the partition communicator (comm.cu): TCP bootstrap + blob all-gather.
#pragma once
#include <cstddef>
#include <cstdint>
#include <string>
#include <vector>

namespace sg {

struct Comm {
    int nranks = 1, rank = 0, device = 0;
    std::vector<int> fds;   // rank 0: one socket per peer (index = rank); others: fds[0] = rank 0
};

// rank 0: open the listening socket, write the 128-byte id
int comm_create_id(uint8_t id[128], std::string &err);
// connect this rank (blocking until every rank has joined, 120 s timeout)
int comm_connect(Comm *c, const uint8_t id[128], int nranks, int rank, std::string &err);
// recv[r * bytes ...] = rank r's `send` (blocking collective)
int comm_allgather(Comm *c, const void *send, void *recv, size_t bytes, std::string &err);
void comm_close(Comm *c);

}  // namespace sg
