// comm.cu — the communicator of the 1-D destination partition (SURVEY.md §8(b) comm_unique_id /
// comm_init / comm_free, §8(e)): a TCP bootstrap between the ranks of one node, used only on the
// host at graph-load time to all-gather small blobs (partition bounds, CUDA IPC handles of each
// rank's exchange arena).  The per-superstep exchange itself never goes through the host: it is
// the peer-memory epilogue of the output kernels (xchg.cuh).
//
// Bootstrap: comm_unique_id (rank 0) opens a listening socket and encodes {magic, nonce, port} in
// the 128-byte id, which the caller broadcasts (e.g. with torch.distributed); comm_init connects
// every rank r > 0 to rank 0 (star).  allgather = every rank sends its blob to rank 0, rank 0
// returns the concatenation.  Address: 127.0.0.1 unless SG_COMM_ADDR names rank 0's IPv4
// address (the partition spans the GPUs of one node).
#include <arpa/inet.h>
#include <netinet/in.h>
#include <netinet/tcp.h>
#include <sys/socket.h>
#include <poll.h>
#include <unistd.h>
#include <cerrno>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <random>
#include <thread>
#include <vector>

#include "comm.h"

namespace sg {

namespace {
constexpr uint32_t kMagic = 0x53474331u;   // "SGC1"
struct IdBlob {
    uint32_t magic;
    uint32_t addr;        // IPv4, network order
    uint16_t port;        // network order
    uint16_t pad;
    uint64_t nonce;
};
static_assert(sizeof(IdBlob) <= 128, "id blob");

// listening sockets opened by comm_unique_id in this process, by nonce (consumed by comm_init)
std::mutex g_mu;
std::vector<std::pair<uint64_t, int>> g_listen;

bool send_all(int fd, const void *p, size_t n) {
    const char *c = static_cast<const char *>(p);
    while (n) {
        const ssize_t k = ::send(fd, c, n, MSG_NOSIGNAL);
        if (k < 0 && errno == EINTR) continue;
        if (k <= 0) return false;
        c += k;
        n -= (size_t)k;
    }
    return true;
}
bool recv_all(int fd, void *p, size_t n, int timeout_ms) {
    char *c = static_cast<char *>(p);
    while (n) {
        pollfd pf{fd, POLLIN, 0};
        const int r = ::poll(&pf, 1, timeout_ms);
        if (r < 0 && errno == EINTR) continue;
        if (r <= 0) return false;
        const ssize_t k = ::recv(fd, c, n, 0);
        if (k < 0 && errno == EINTR) continue;
        if (k <= 0) return false;
        c += k;
        n -= (size_t)k;
    }
    return true;
}
uint32_t bootstrap_addr() {
    const char *e = getenv("SG_COMM_ADDR");
    in_addr a{};
    if (e && inet_pton(AF_INET, e, &a) == 1) return a.s_addr;
    return htonl(INADDR_LOOPBACK);
}
}  // namespace

int comm_create_id(uint8_t id[128], std::string &err) {
    memset(id, 0, 128);
    const int fd = ::socket(AF_INET, SOCK_STREAM, 0);
    if (fd < 0) {
        err = "socket() failed";
        return -1;
    }
    int one = 1;
    setsockopt(fd, SOL_SOCKET, SO_REUSEADDR, &one, sizeof one);
    sockaddr_in sa{};
    sa.sin_family = AF_INET;
    sa.sin_addr.s_addr = htonl(INADDR_ANY);
    sa.sin_port = 0;
    if (::bind(fd, reinterpret_cast<sockaddr *>(&sa), sizeof sa) != 0 || ::listen(fd, 64) != 0) {
        ::close(fd);
        err = "bind/listen failed";
        return -1;
    }
    socklen_t len = sizeof sa;
    getsockname(fd, reinterpret_cast<sockaddr *>(&sa), &len);
    IdBlob b{};
    b.magic = kMagic;
    b.addr = bootstrap_addr();
    b.port = sa.sin_port;
    std::random_device rd;
    b.nonce = ((uint64_t)rd() << 32) ^ rd() ^ (uint64_t)std::chrono::steady_clock::now().time_since_epoch().count();
    memcpy(id, &b, sizeof b);
    std::lock_guard<std::mutex> lk(g_mu);
    g_listen.emplace_back(b.nonce, fd);
    return 0;
}

int comm_connect(Comm *c, const uint8_t id[128], int nranks, int rank, std::string &err) {
    IdBlob b;
    memcpy(&b, id, sizeof b);
    if (b.magic != kMagic) {
        err = "not a sygraph communicator id";
        return -1;
    }
    c->nranks = nranks;
    c->rank = rank;
    c->fds.assign(nranks, -1);
    const int timeout_ms = 120000;
    if (rank == 0) {
        int lfd = -1;
        {
            std::lock_guard<std::mutex> lk(g_mu);
            for (size_t i = 0; i < g_listen.size(); i++)
                if (g_listen[i].first == b.nonce) {
                    lfd = g_listen[i].second;
                    g_listen.erase(g_listen.begin() + (long)i);
                    break;
                }
        }
        if (lfd < 0) {
            err = "rank 0 must call comm_init with the id its own comm_unique_id created";
            return -1;
        }
        for (int got = 1; got < nranks;) {
            pollfd pf{lfd, POLLIN, 0};
            if (::poll(&pf, 1, timeout_ms) <= 0) {
                ::close(lfd);
                err = "timed out waiting for peers to connect";
                return -1;
            }
            const int fd = ::accept(lfd, nullptr, nullptr);
            if (fd < 0) continue;
            int one = 1;
            setsockopt(fd, IPPROTO_TCP, TCP_NODELAY, &one, sizeof one);
            uint64_t hello[2];
            if (!recv_all(fd, hello, sizeof hello, timeout_ms) || hello[0] != b.nonce || hello[1] == 0 ||
                hello[1] >= (uint64_t)nranks || c->fds[hello[1]] >= 0) {
                ::close(fd);
                continue;
            }
            c->fds[hello[1]] = fd;
            got++;
        }
        ::close(lfd);
    } else {
        sockaddr_in sa{};
        sa.sin_family = AF_INET;
        sa.sin_addr.s_addr = b.addr;
        sa.sin_port = b.port;
        const auto t0 = std::chrono::steady_clock::now();
        int fd = -1;
        for (;;) {
            fd = ::socket(AF_INET, SOCK_STREAM, 0);
            if (fd >= 0 && ::connect(fd, reinterpret_cast<sockaddr *>(&sa), sizeof sa) == 0) break;
            if (fd >= 0) ::close(fd);
            fd = -1;
            if (std::chrono::steady_clock::now() - t0 > std::chrono::milliseconds(timeout_ms)) break;
            std::this_thread::sleep_for(std::chrono::milliseconds(20));
        }
        if (fd < 0) {
            err = "could not connect to rank 0";
            return -1;
        }
        int one = 1;
        setsockopt(fd, IPPROTO_TCP, TCP_NODELAY, &one, sizeof one);
        const uint64_t hello[2] = {b.nonce, (uint64_t)rank};
        if (!send_all(fd, hello, sizeof hello)) {
            ::close(fd);
            err = "send to rank 0 failed";
            return -1;
        }
        c->fds[0] = fd;
    }
    return 0;
}

int comm_allgather(Comm *c, const void *send, void *recv, size_t bytes, std::string &err) {
    char *out = static_cast<char *>(recv);
    const int timeout_ms = 300000;
    if (c->nranks <= 1) {
        memmove(out, send, bytes);
        return 0;
    }
    if (c->rank == 0) {
        memmove(out, send, bytes);
        for (int r = 1; r < c->nranks; r++)
            if (!recv_all(c->fds[r], out + (size_t)r * bytes, bytes, timeout_ms)) {
                err = "allgather: receive from a peer failed";
                return -1;
            }
        for (int r = 1; r < c->nranks; r++)
            if (!send_all(c->fds[r], out, bytes * (size_t)c->nranks)) {
                err = "allgather: send to a peer failed";
                return -1;
            }
    } else {
        if (!send_all(c->fds[0], send, bytes) || !recv_all(c->fds[0], out, bytes * (size_t)c->nranks, timeout_ms)) {
            err = "allgather: exchange with rank 0 failed";
            return -1;
        }
    }
    return 0;
}

void comm_close(Comm *c) {
    for (int fd : c->fds)
        if (fd >= 0) ::close(fd);
    c->fds.clear();
}

}  // namespace sg
